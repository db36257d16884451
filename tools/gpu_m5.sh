#!/bin/bash
O=gpurun_out/${TAG:-m5}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log; tail -3 $O/gputest.log
GPL_DEBUG_TUNE=1 GPL_DEBUG_MODEL=1 timeout 2400 python experiments.py model > $O/model.log 2>&1; cp gpurun_out/model_vs_autotune_sf100.json $O/; tail -c 300 $O/model.log
GPL_DEBUG_MODEL=1 timeout 1500 python experiments.py knobs > $O/knobs.log 2>&1; cp gpurun_out/knob_sweep_config2.json $O/; tail -c 600 $O/knobs.log
