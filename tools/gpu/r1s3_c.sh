make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 600 python -m pytest tests -m gpu -x -q -k "gamma or autotune" > gpurun_out/pytest_gpu_c.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu_c.log
timeout -s KILL 900 python experiments.py gamma > gpurun_out/gamma.log 2>&1; echo "gamma rc=$?"; tail -c 3000 gpurun_out/gamma.log
timeout -s KILL 600 python experiments.py warps > gpurun_out/warps.log 2>&1; echo "warps rc=$?"; tail -c 1500 gpurun_out/warps.log
