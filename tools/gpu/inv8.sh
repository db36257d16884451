make -j16 > gpurun_out/make.log 2>&1
timeout 300 python tools/host_overhead.py Q5 1 > gpurun_out/host_q5.log 2>&1
GPL_NO_COPYOUT=1 timeout 300 python tools/host_overhead.py Q5 1 > gpurun_out/host_q5_nocopy.log 2>&1
cat gpurun_out/host_q5.log gpurun_out/host_q5_nocopy.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_q5_sf1.csv python tools/step_once.py Q5 1 2 > gpurun_out/launch_q5_sf1.log 2>&1
GPL_NO_COPYOUT=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_q5_sf1_nocopy.csv python tools/step_once.py Q5 1 2 > gpurun_out/launch_q5_sf1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_q5_sf5.csv python tools/step_once.py Q5 5 1 > gpurun_out/launch_q5_sf5.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python tools/plan_variants.py Q5 20 > gpurun_out/variants_Q5.log 2>&1
