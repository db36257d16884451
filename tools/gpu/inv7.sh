make -j16 > gpurun_out/make.log 2>&1
timeout 300 python tools/host_overhead.py Q5 1 > gpurun_out/host_q5.log 2>&1
cat gpurun_out/host_q5.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_q5_sf1.csv python tools/step_once.py Q5 1 2 > gpurun_out/launch_q5_sf1.log 2>&1
timeout 900 python tools/build_shapes.py Q5 5 > gpurun_out/build_shapes_q5.log 2>&1
timeout 600 python tools/plan_variants.py Q5 1 > gpurun_out/variants_Q5_sf1.log 2>&1
timeout 600 python tools/plan_variants.py Q5 20 > gpurun_out/variants_Q5.log 2>&1
timeout 600 python tools/plan_variants.py Q7 20 > gpurun_out/variants_Q7.log 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
