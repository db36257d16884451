#!/bin/bash
# SF 100 round trip: the default bench line, JIT kernel dumps (SASS inspection),
# an ncu --set full capture of one query step, and the full-size parity record.
# usage: bash tools/gpu_sf100.sh TAG [queries...]
TAG=${1:-r2}; shift
QS=${@:-Q5 Q7}
O=gpurun_out/$TAG; mkdir -p $O/jit
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > $O/bench_q5_sf100.json 2> $O/bench_q5_sf100.err
for q in $QS; do
  GPL_JIT_DUMP=$O/jit timeout 600 python tools/step_once.py $q 100 1 > $O/step_$q.txt 2>&1
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:gpl_pipeline_jit -c 24 \
      -o $O/ncu_$q python tools/step_once.py $q 100 1 > $O/ncu_$q.log 2>&1
done
timeout 3000 python tools/verify_sf100.py $O/verify_sf100.json 100 > $O/verify.log 2>&1
tail -2 $O/verify.log; cat $O/bench_q5_sf100.json | head -c 600
