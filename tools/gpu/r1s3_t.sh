mkdir -p gpurun_out/dr; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 600 python -m pytest tests -m gpu -x -q -k "drain and jit" > gpurun_out/pytest_gpu_t.log 2>&1; echo "pytest-drain rc=$?"; tail -30 gpurun_out/pytest_gpu_t.log
