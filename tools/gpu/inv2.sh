make -j16 > gpurun_out/make.log 2>&1
GPL_TRACE_HOST=1 timeout 300 python tools/step_breakdown.py Q5 1 > gpurun_out/step_q5_trace.log 2>&1
for q in Q8 Q5 Q7; do timeout 600 python tools/plan_variants.py $q 20 > gpurun_out/variants_$q.log 2>&1; done
