make -j16 > gpurun_out/make.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
timeout 300 python tools/host_overhead.py Q5 1 > gpurun_out/host_q5.log 2>&1
cat gpurun_out/host_q5.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_q5_sf1.csv python tools/step_once.py Q5 1 2 > gpurun_out/launch_q5_sf1.log 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
bash tools/gpu/sf100.sh
