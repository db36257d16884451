#!/bin/bash
# Experiments round trip: GPL (w/o CE) tests, config 5 (fused vs KBE vs GPL w/o CE, SF 10), config 2 knob
# sweep (SF 1 Q5: s x n x Δ), the A9 model pick vs autotune (SF 100), and ncu source captures.
TAG=${1:-exp}; shift
O=gpurun_out/$TAG; mkdir -p $O
timeout 600 python -m pytest tests -m gpu -q -k "without_ce or kbe" > $O/gputest_kbe.log 2>&1; tail -2 $O/gputest_kbe.log
timeout 1200 python experiments.py kbe > $O/kbe.log 2>&1; cp gpurun_out/kbe_config5.json $O/ 2>/dev/null; tail -c 300 $O/kbe.log
timeout 1500 python experiments.py knobs > $O/knobs.log 2>&1; cp gpurun_out/knob_sweep_config2.json $O/ 2>/dev/null; tail -c 600 $O/knobs.log
timeout 2400 python experiments.py model > $O/model.log 2>&1; cp gpurun_out/model_vs_autotune_sf100.json $O/ 2>/dev/null; tail -c 800 $O/model.log
[ -n "$NCU_QS" ] && bash tools/gpu_ncu.sh $TAG $NCU_QS
