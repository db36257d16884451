#!/bin/bash
O=gpurun_out/${TAG:-m4}; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "autotune or gamma or profiled or dense_warp or knob or schedule" > $O/gputest.log 2>&1; tail -2 $O/gputest.log
for i in 1 2; do
timeout 300 python tools/dense_groups.py 10 build/old/libgpl.so >> $O/dense.log 2>&1
timeout 300 python tools/dense_groups.py 10 >> $O/dense.log 2>&1
done
cut -c1-300 $O/dense.log
GPL_DEBUG_TUNE=1 GPL_DEBUG_MODEL=1 timeout 2400 python experiments.py model > $O/model.log 2>&1; cp gpurun_out/model_vs_autotune_sf100.json $O/; tail -c 300 $O/model.log
GPL_DEBUG_MODEL=1 timeout 1500 python experiments.py knobs > $O/knobs.log 2>&1; cp gpurun_out/knob_sweep_config2.json $O/; tail -c 600 $O/knobs.log
