#!/bin/bash
# GPU suite + per-query bench lines (model shape) + Q5 with gpl_autotune + the default bench line
O=gpurun_out/${TAG:-b1}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log; tail -3 $O/gputest.log
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err
python - <<PY
import json; b = json.loads(open("$O/bench.json").read().strip().splitlines()[-1])
print("default", b["value"], b["ms_per_step"], b["kernel_ms"], b["roofline"]["frac"], b["config"]["shape"], b["e2e"]["ms_per_step"], b["clocks"])
PY
for q in Q5 Q7 Q8 Q9 Q14 Q3; do
  for sh in model autotune; do
    if [ $sh = autotune ] && [ $q != Q5 ] && [ $q != Q9 ]; then continue; fi
    timeout 900 python bench.py --query $q --shape $sh --no-e2e --no-cpu-baseline --steps 30 > $O/bench_${q}_$sh.json 2> $O/bench_${q}_$sh.err
    python - <<PY
import json; b = json.loads(open("$O/bench_${q}_$sh.json").read().strip().splitlines()[-1])
print("$q", "$sh", round(b["ms_per_step"], 4), round(b["kernel_ms"], 4), round(b["roofline"]["frac"], 3), b["roofline"]["bytes_per_launch"])
PY
  done
done
