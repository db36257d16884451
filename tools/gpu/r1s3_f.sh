make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 900 python -m pytest tests -m gpu -x -q -k "q3 or profiled or gamma" > gpurun_out/pytest_gpu_f.log 2>&1; echo "pytest-q3 rc=$?"; tail -30 gpurun_out/pytest_gpu_f.log
timeout -s KILL 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_f2.log 2>&1; echo "pytest-all rc=$?"; tail -5 gpurun_out/pytest_gpu_f2.log
