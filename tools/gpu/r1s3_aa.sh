mkdir -p gpurun_out/ls2; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 1500 python -m pytest tests -m gpu -x -q > gpurun_out/ls2/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/ls2/pytest.log
timeout -s KILL 600 python bench.py > gpurun_out/ls2/q5_sf1.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/ls2/q5_sf1.json'));print('Q5 sf1', d['ms_per_step'],d['kernel_ms'],d['roofline']['frac'],d['pipeline'])"
for q in Q7 Q5 Q9 Q3; do
timeout -s KILL 900 python bench.py --query $q --sf 100 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ls2/$q.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/ls2/$q.json'));print('$q', d['ms_per_step'],d['kernel_ms'],d['roofline']['frac'],d['pipeline'])"
done
