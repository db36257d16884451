#!/bin/bash
# ncu --set full (with source) of one warm query step per query at SF (default 100), exported to CSV on the
# box (raw / details / SASS source pages); the .ncu-rep comes back only when small.
# usage: bash tools/gpu_ncu.sh TAG Q...   (GPL_OPTS pins options after the autotune)
TAG=${1:-ncu}; shift
O=gpurun_out/$TAG; mkdir -p $O/jit
for q in "$@"; do
  GPL_JIT_DUMP=$O/jit timeout 600 python tools/ncu_probe.py $q ${SF:-100} > $O/step_$q.txt 2>&1; tail -1 $O/step_$q.txt
  timeout 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:gpl_pipeline_jit \
      -o /tmp/ncu_$q python tools/ncu_probe.py $q ${SF:-100} > $O/ncu_$q.log 2>&1
  ncu -i /tmp/ncu_$q.ncu-rep --page details --csv > $O/ncu_details_$q.csv 2>/dev/null
  ncu -i /tmp/ncu_$q.ncu-rep --page source --csv --print-source sass > $O/ncu_sass_$q.csv 2>/dev/null
  sz=$(stat -c %s /tmp/ncu_$q.ncu-rep 2>/dev/null || echo 0)
  if [ "$sz" -lt 12000000 ]; then cp /tmp/ncu_$q.ncu-rep $O/; fi
done
du -sh $O
