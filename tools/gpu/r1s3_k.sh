mkdir -p gpurun_out/q3; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/q3/launches_q3_sf10_v2.csv python bench.py --query Q3 --sf 10 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu-list rc=$?"
timeout -s KILL 600 python bench.py --query Q3 --sf 10 --steps 10 --no-cpu-baseline > gpurun_out/q3/bench_q3_sf10_v2.json 2> /dev/null; echo "bench rc=$?"; cat gpurun_out/q3/bench_q3_sf10_v2.json
