set -x
make -j16 > gpurun_out/make.log 2>&1
timeout 300 python tools/step_breakdown.py Q5 1 > gpurun_out/step_q5.log 2>&1
timeout 600 python tools/try_shapes.py Q8 20 1024,3,4,2 2048,3,4,2 1024,3,8,1 1024,3,8,2 512,4,8,2 1024,3,12,1 1024,3,16,1 2048,2,16,1 > gpurun_out/shapes_q8.log 2>&1
timeout 600 python tools/try_shapes.py Q5 20 1024,3,4,2 1024,3,8,1 1024,3,8,2 512,4,8,2 1024,3,12,1 1024,3,16,1 > gpurun_out/shapes_q5.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:gpl_pipeline -s 3 -c 1 -o gpurun_out/q8_sf20 -f python tools/try_shapes.py Q8 20 1024,3,4,2 > gpurun_out/ncu_q8.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:gpl_pipeline -s 3 -c 1 -o gpurun_out/q5_sf20 -f python tools/try_shapes.py Q5 20 1024,3,4,2 > gpurun_out/ncu_q5.log 2>&1
ls -la gpurun_out
