#!/bin/bash
# Validation round trip: the whole GPU suite (no -x), smoke, compute-sanitizer memcheck / synccheck /
# racecheck over every kernel variant (tools/sanitize_run.py), and the config-5 fused vs KBE vs GPL (w/o CE)
# experiment. usage: bash tools/gpu_validate.sh TAG
TAG=${1:-val}
O=gpurun_out/$TAG; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log
tail -4 $O/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
tail -2 $O/smoke.log
for tool in memcheck synccheck racecheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 200 python tools/sanitize_run.py > $O/sanitizer_$tool.log 2>&1
  echo "$tool rc=$?" >> $O/sanitizer_$tool.log
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|rc=|MISMATCH" $O/sanitizer_$tool.log | tail -4
done
timeout 1200 python experiments.py kbe > $O/kbe.log 2>&1; tail -c 600 $O/kbe.log
cp gpurun_out/kbe_config5.json $O/ 2>/dev/null
