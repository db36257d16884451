mkdir -p gpurun_out/dr; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_u.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/pytest_gpu_u.log
GPL_DEBUG_TUNE=1 timeout -s KILL 600 python bench.py > gpurun_out/dr/q5_sf1.json 2> gpurun_out/dr/q5_sf1.err; python -c "import json;d=json.load(open('gpurun_out/dr/q5_sf1.json'));print('Q5 sf1', d['ms_per_step'],d['kernel_ms'],d['pipeline'])"; grep "autotune: split" gpurun_out/dr/q5_sf1.err | sort -t: -k3 -n | head -4
for q in Q7 Q5 Q8 Q3; do
GPL_DEBUG_TUNE=1 timeout -s KILL 900 python bench.py --query $q --sf 100 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/dr/$q.json 2> gpurun_out/dr/$q.err; python -c "import json;d=json.load(open('gpurun_out/dr/$q.json'));print('$q', d['ms_per_step'],d['kernel_ms'],d['pipeline'])"; grep "autotune: split" gpurun_out/dr/$q.err | sort -t: -k3 -n | head -5
done
