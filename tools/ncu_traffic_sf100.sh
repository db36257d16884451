#!/bin/bash
# Per-launch DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum) of the
# fused probe kernel of bench.py's timed step at SF 100, one query per run.
# The last gpl_pipeline_jit launch of a --steps 1 run is the timed step's probe
# kernel (graph replay; e2e off). Output: gpurun_out/traffic/<Q>_sf100.csv
mkdir -p gpurun_out/traffic
for q in "$@"; do
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none -k regex:gpl_pipeline_jit --csv \
    --log-file gpurun_out/traffic/${q}_sf100.csv \
    python bench.py --query $q --sf 100 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
    > gpurun_out/traffic/${q}_sf100.log 2>&1
  echo "$q exit $?"
done
