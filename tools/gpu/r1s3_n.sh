mkdir -p gpurun_out/sf100_v4; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 600 python -m pytest tests -m gpu -q -k "profiled" > gpurun_out/pytest_gpu_n.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/pytest_gpu_n.log
for q in Q14 Q5 Q7 Q8 Q9 Q3; do
  timeout -s KILL 900 python bench.py --query $q --sf 100 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/sf100_v4/$q.json 2> gpurun_out/sf100_v4/$q.err
  echo "$q rc=$?"; python -c "import json;d=json.load(open('gpurun_out/sf100_v4/$q.json'));print(d['ms_per_step'],d['kernel_ms'],d['roofline']['frac'],d['roofline']['moved_gbs'],d['e2e']['ms_per_step'])"
done
timeout -s KILL 600 python bench.py --query Q9 --sf 10 --steps 10 > gpurun_out/sf100_v4/Q9_sf10.json 2> gpurun_out/sf100_v4/Q9_sf10.err; echo "Q9 sf10 rc=$?"
