#!/bin/bash
O=gpurun_out/f3; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log; tail -3 $O/gputest.log
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; python -c "import json; b=json.load(open('$O/bench.json')); print(b['kernel_ms'], b['ms_per_step'], b['roofline']['frac'], b['clocks'], b['e2e']['ms_per_step'])"
bash tools/gpu_perf.sh f3 Q5 Q9 Q14
