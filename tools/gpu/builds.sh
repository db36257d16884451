make -j16 > gpurun_out/make.log 2>&1
mkdir -p gpurun_out/bl
for o in "" "consumer_warps=16" "consumer_warps=16,packets=2" "consumer_warps=8,ctas_per_sm=2" "consumer_warps=8,ctas_per_sm=2,packets=2" "consumer_warps=16,stage_rows=512" "consumer_warps=16,stage_rows=512,packets=2" "consumer_warps=12,stage_rows=1024,ring_depth=4,packets=2"; do
  n=$(echo "x$o" | tr ',=' '__')
  GPL_OPTS="$o" timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bl/$n.csv python tools/step_once.py Q5 1 1 > gpurun_out/bl/$n.log 2>&1
  echo "$o: $(grep gpl_pipeline_jit gpurun_out/bl/$n.csv | tail -4 | awk -F'","' '{print $NF}' | tr -d '"' | tr '\n' ' ')"
done
