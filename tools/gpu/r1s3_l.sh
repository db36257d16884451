mkdir -p gpurun_out/q3; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 900 python -m pytest tests -m gpu -x -q -k "q3" > gpurun_out/pytest_gpu_l.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_l.log
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/q3/launches_q3_sf10_v4.csv python bench.py --query Q3 --sf 10 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu-list rc=$?"
timeout -s KILL 600 python bench.py --query Q3 --sf 10 --steps 10 --no-cpu-baseline > gpurun_out/q3/bench_q3_sf10_v4.json 2> gpurun_out/q3/bench_q3_sf10_v4.err; echo "bench rc=$?"; cat gpurun_out/q3/bench_q3_sf10_v4.json; grep autotune: gpurun_out/q3/bench_q3_sf10_v4.err | sort -t: -k3 -n | head -12
