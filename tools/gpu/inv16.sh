make -j16 > gpurun_out/make.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
timeout 900 ncu --set full --import-source on --clock-control none -k regex:gpl_pipeline --launch-skip 19 --launch-count 1 -o gpurun_out/probe_q5_sf1_lazy -f python tools/step_once.py Q5 1 4 > gpurun_out/ncu_probe.log 2>&1; echo "ncu rc=$?"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_q5_sf1.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1; echo "ncu-bench rc=$?"
