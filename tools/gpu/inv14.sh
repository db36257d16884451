make -j16 > gpurun_out/make.log 2>&1
timeout 600 python tools/knob_check.py 1 > gpurun_out/knob_all.log 2>&1; echo "knobs rc=$?"; tail -2 gpurun_out/knob_all.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python tools/try_shapes.py Q5 1 1024,3,4,2,1,1 1024,3,4,2,2,1 2048,3,8,1,1,1 2048,3,8,1,2,1 1024,4,12,1,2,1 > gpurun_out/shapes_q5_sf1.log 2>&1
cat gpurun_out/shapes_q5_sf1.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
