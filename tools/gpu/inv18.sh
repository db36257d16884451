make -j16 > gpurun_out/make.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bl/new.csv python tools/step_once.py Q5 1 1 > /dev/null 2>&1
echo "builds: $(grep -E 'gpl_pipeline_jit|clear|copyout' gpurun_out/bl/new.csv | tail -6 | awk -F'","' '{print $NF}' | tr -d '"' | tr '\n' ' ')"
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
