#!/bin/bash
# SF 100 round trip: the default bench line, JIT kernel dumps (SASS inspection),
# ncu of one warm query step (launch list + --set full of its kernels, exported
# to CSV on the box so only small files come back), and the full-size parity record.
# usage: bash tools/gpu_sf100.sh TAG [queries...]
TAG=${1:-r2}; shift
QS=${@:-Q5 Q7}
O=gpurun_out/$TAG; mkdir -p $O/jit
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > $O/bench_q5_sf100.json 2> $O/bench_q5_sf100.err
for q in $QS; do
  GPL_JIT_DUMP=$O/jit timeout 600 python tools/ncu_probe.py $q 100 > $O/step_$q.txt 2>&1
  timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
      --clock-control none --csv python tools/ncu_probe.py $q 100 > $O/launches_$q.csv 2> $O/launches_$q.err
  timeout 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:gpl_pipeline_jit \
      -o /tmp/ncu_$q python tools/ncu_probe.py $q 100 > $O/ncu_$q.log 2>&1
  ncu -i /tmp/ncu_$q.ncu-rep --page raw --csv > $O/ncu_raw_$q.csv 2>/dev/null
  ncu -i /tmp/ncu_$q.ncu-rep --page details --csv > $O/ncu_details_$q.csv 2>/dev/null
  ncu -i /tmp/ncu_$q.ncu-rep --page source --csv --print-source sass > $O/ncu_sass_$q.csv 2>/dev/null
  sz=$(stat -c %s /tmp/ncu_$q.ncu-rep 2>/dev/null || echo 0)
  if [ "$sz" -lt 12000000 ]; then cp /tmp/ncu_$q.ncu-rep $O/; fi
done
[ "$SKIP_VERIFY" = "1" ] || timeout 3000 python tools/verify_sf100.py $O/verify_sf100.json 100 > $O/verify.log 2>&1
du -sh $O; tail -2 $O/verify.log; head -c 400 $O/bench_q5_sf100.json
