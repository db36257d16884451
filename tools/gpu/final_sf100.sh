# config 4 (1 GPU): every paper query at SF 100 + config 3 (Q9 SF 10) + config 5 (KBE) + verification
make -j16 > gpurun_out/make.log 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "reload or late_mat or pipelined_build" > gpurun_out/pytest_gpu3.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu3.log
mkdir -p gpurun_out/bl
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bl/new.csv python tools/step_once.py Q5 1 1 > /dev/null 2>&1
echo "launches: $(grep -E 'gpl_pipeline_jit|clear|copyout' gpurun_out/bl/new.csv | tail -6 | awk -F'","' '{print $NF}' | tr -d '"' | tr '\n' ' ')"
mkdir -p gpurun_out/sf100
for q in Q14 Q5 Q7 Q8 Q9; do
  timeout 900 python bench.py --query $q --sf 100 --steps 10 --warmup 3 > gpurun_out/sf100/$q.json 2> gpurun_out/sf100/$q.err
  echo "$q rc=$?"
done
timeout 600 python bench.py --query Q9 --sf 10 > gpurun_out/sf100/Q9_sf10.json 2> gpurun_out/sf100/Q9_sf10.err
timeout 1800 python experiments.py kbe > gpurun_out/kbe.log 2>&1; echo "kbe rc=$?"
timeout 1500 python tools/verify_sf100.py gpurun_out/verify_sf100_r01c.json 100 > gpurun_out/verify.log 2>&1; echo "verify rc=$?"
