#!/bin/bash
O=gpurun_out/${TAG:-knobs}; mkdir -p $O
GPL_DEBUG_MODEL=1 timeout 1500 python experiments.py knobs > $O/knobs.log 2>&1; cp gpurun_out/knob_sweep_config2.json $O/; tail -c 600 $O/knobs.log; grep "^apply_profile" $O/knobs.log | sort | uniq -c | head
