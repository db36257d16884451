#!/bin/bash
# Kernel iteration loop on the GPU box: GPU tests (optional), then for each query at SF 100 the
# autotuned probe kernel time and an ncu instruction/duration/DRAM summary of one warm step.
# usage: TESTS=1 bash tools/gpu_perf.sh TAG Q5 Q7 ...
TAG=${1:-perf}; shift
QS=${@:-Q5 Q7}
O=gpurun_out/$TAG; mkdir -p $O
if [ "$TESTS" = "1" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log
  tail -3 $O/gputest.log
fi
for q in $QS; do
  timeout 600 python tools/ncu_probe.py $q ${SF:-100} > $O/step_$q.txt 2>&1; tail -1 $O/step_$q.txt
  timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active \
      --clock-control none --csv python tools/ncu_probe.py $q ${SF:-100} > $O/launches_$q.csv 2> $O/launches_$q.err
  python tools/launch_summary.py $O/launches_$q.csv
done
