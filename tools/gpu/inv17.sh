make -j16 > gpurun_out/make.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:gpl_pipeline --launch-skip 5 --launch-count 1 -o gpurun_out/build_hto_sf1_v2 -f python tools/step_once.py Q5 1 2 > gpurun_out/ncu_build.log 2>&1
GPL_DEBUG_DESC=1 timeout 300 python tools/step_once.py Q5 1 1 > gpurun_out/desc.log 2>&1
