#!/bin/bash
# A9 model checks: config-2 knob sweep (Eq 10 error) and the model's own pick vs gpl_autotune at SF 100.
TAG=${1:-model}
O=gpurun_out/$TAG; mkdir -p $O
timeout 1500 python experiments.py knobs > $O/knobs.log 2>&1; cp gpurun_out/knob_sweep_config2.json $O/; tail -c 600 $O/knobs.log; echo
GPL_DEBUG_MODEL=1 timeout 2400 python experiments.py model > $O/model.log 2>&1; cp gpurun_out/model_vs_autotune_sf100.json $O/; tail -c 600 $O/model.log
