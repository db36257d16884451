make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_j.log 2>&1; echo "pytest-all rc=$?"; tail -25 gpurun_out/pytest_gpu_j.log
bash tools/gpu/r1s3_i.sh
