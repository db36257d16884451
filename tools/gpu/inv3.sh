make -j16 > gpurun_out/make.log 2>&1
timeout 300 python tools/host_overhead.py Q5 1 > gpurun_out/host_q5.log 2>&1
timeout 300 python tools/host_overhead.py Q5 1 > gpurun_out/host_q5.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_gpu.log
GPL_BUILD_PIPE=1 timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json
for q in Q8 Q5 Q7; do timeout 600 python tools/plan_variants.py $q 20 > gpurun_out/variants_$q.log 2>&1; done
