make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
GPL_DEBUG_MODEL=1 timeout -s KILL 900 python -m pytest tests -m gpu -x -q -k "profiled" > gpurun_out/pytest_gpu_g0.log 2>&1; echo "pytest-prof rc=$?"; grep -a "apply_profile" gpurun_out/pytest_gpu_g0.log | head; tail -5 gpurun_out/pytest_gpu_g0.log
timeout -s KILL 900 python -m pytest tests -m gpu -x -q -k "q3" > gpurun_out/pytest_gpu_g.log 2>&1; echo "pytest-q3 rc=$?"; tail -30 gpurun_out/pytest_gpu_g.log
