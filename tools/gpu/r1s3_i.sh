# Q3 (NEXT-4) measurement: bench SF 10 / SF 100, launch list, ncu full capture of the fused kernel and the
# selection kernels, SF 100 verification; Q5 SF 1 default bench with the widened autotune
make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
mkdir -p gpurun_out/q3
timeout -s KILL 600 python bench.py > gpurun_out/q3/bench_q5_sf1.json 2> gpurun_out/q3/bench_q5_sf1.err; echo "bench q5 rc=$?"; cat gpurun_out/q3/bench_q5_sf1.json
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/q3/launches_q3_sf10.csv python bench.py --query Q3 --sf 10 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu-list rc=$?"
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:"pipeline|select_phase" -s 6 -c 3 -o gpurun_out/q3/prof_q3_sf10 python bench.py --query Q3 --sf 10 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-autotune > gpurun_out/q3/ncu_full.log 2>&1; echo "ncu-full rc=$?"; tail -2 gpurun_out/q3/ncu_full.log
timeout -s KILL 900 python bench.py --query Q3 --sf 100 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/q3/bench_q3_sf100.json 2> gpurun_out/q3/bench_q3_sf100.err; echo "bench q3 sf100 rc=$?"; cat gpurun_out/q3/bench_q3_sf100.json
timeout -s KILL 1500 python tools/verify_q3.py gpurun_out/q3/verify_q3_sf100.json 100 > gpurun_out/q3/verify.log 2>&1; echo "verify rc=$?"; tail -3 gpurun_out/q3/verify.log
