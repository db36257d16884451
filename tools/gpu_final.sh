#!/bin/bash
# Final round trip: the whole GPU suite, smoke, the default bench line (+ the reference arm), the
# full-size SF 100 parity record, and the model experiments.
TAG=${1:-final}
O=gpurun_out/$TAG; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log; tail -3 $O/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; head -c 300 $O/bench.json; echo
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; head -c 200 $O/bench_ref.json; echo
timeout 3000 python tools/verify_sf100.py $O/verify_sf100.json 100 > $O/verify.log 2>&1; tail -3 $O/verify.log
[ "$EXPS" = "1" ] && { timeout 1500 python experiments.py knobs > $O/knobs.log 2>&1; cp gpurun_out/knob_sweep_config2.json $O/; tail -c 400 $O/knobs.log; timeout 2400 python experiments.py model > $O/model.log 2>&1; cp gpurun_out/model_vs_autotune_sf100.json $O/; tail -c 400 $O/model.log; }
