make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_fin2.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_fin2.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_fin2.log 2>&1; echo "smoke rc=$?"; tail -4 gpurun_out/smoke_fin2.log
