make -j16 > gpurun_out/make.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:gpl_pipeline --launch-skip 1 --launch-count 1 -o gpurun_out/build_hto_sf1 -f python tools/step_once.py Q5 1 1 > gpurun_out/ncu_build.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:gpl_pipeline --launch-skip 3 --launch-count 1 -o gpurun_out/probe_q5_sf1 -f python tools/step_once.py Q5 1 1 > gpurun_out/ncu_probe.log 2>&1
