make -j16 > gpurun_out/make.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python tools/lazy_compare.py 20 Q5,Q8,Q7 > gpurun_out/cl_sf20.log 2>&1; cat gpurun_out/cl_sf20.log
timeout 600 python tools/lazy_compare.py 1 Q5 > gpurun_out/cl_sf1.log 2>&1; cat gpurun_out/cl_sf1.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
