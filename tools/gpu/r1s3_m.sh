mkdir -p gpurun_out/q3; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_m.log 2>&1; echo "pytest rc=$?"; tail -8 gpurun_out/pytest_gpu_m.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
timeout -s KILL 600 python bench.py > gpurun_out/bench_m.json 2> gpurun_out/bench_m.err; echo "bench rc=$?"; cat gpurun_out/bench_m.json
