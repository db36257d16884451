#!/bin/bash
O=gpurun_out/f2; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q -k "parity_small or finalize or partitioned or qf or gamma" > $O/gputest.log 2>&1; tail -2 $O/gputest.log
bash tools/gpu_perf.sh f2 Q5 Q7 Q14 Q8
timeout 600 python tools/h2d_ceiling.py 16327672504 > $O/h2d_ceiling.json 2>&1; cat $O/h2d_ceiling.json
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; python -c "import json; b=json.load(open('$O/bench.json')); print(b['kernel_ms'], b['ms_per_step'], b['roofline']['frac'], b['clocks'], b['e2e']['ms_per_step'])"
timeout 1500 python experiments.py knobs > $O/knobs.log 2>&1; cp gpurun_out/knob_sweep_config2.json $O/; tail -c 300 $O/knobs.log
timeout 2400 python experiments.py model > $O/model.log 2>&1; cp gpurun_out/model_vs_autotune_sf100.json $O/; tail -c 300 $O/model.log
