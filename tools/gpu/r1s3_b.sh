make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 600 python -m pytest tests -m gpu -x -q -k "autotune or build" > gpurun_out/pytest_gpu_b.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_b.log
timeout -s KILL 300 python tools/step_breakdown.py Q5 1 > gpurun_out/breakdown_q5_sf1.log 2>&1; cat gpurun_out/breakdown_q5_sf1.log
timeout -s KILL 600 python bench.py > gpurun_out/bench_b.json 2> gpurun_out/bench_b.err; echo "bench rc=$?"; cat gpurun_out/bench_b.json
timeout -s KILL 600 python bench.py --query Q9 --sf 10 --steps 10 --no-cpu-baseline > gpurun_out/bench_q9_b.json 2> gpurun_out/bench_q9_b.err; echo "bench rc=$?"; cat gpurun_out/bench_q9_b.json
