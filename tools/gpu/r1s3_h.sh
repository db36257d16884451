make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_h.log 2>&1; echo "pytest-all rc=$?"; tail -25 gpurun_out/pytest_gpu_h.log
timeout -s KILL 600 python bench.py --query Q3 --sf 10 --steps 10 --no-cpu-baseline > gpurun_out/bench_q3_sf10.json 2> gpurun_out/bench_q3_sf10.err; echo "bench q3 rc=$?"; cat gpurun_out/bench_q3_sf10.json; tail -3 gpurun_out/bench_q3_sf10.err
