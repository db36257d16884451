#!/bin/bash
O=gpurun_out/m2; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "dense_warp or forced_global or parity_small" > $O/gputest.log 2>&1; tail -2 $O/gputest.log
for i in 1 2; do
timeout 300 python tools/dense_groups.py 10 build/old/libgpl.so >> $O/dense.log 2>&1
timeout 300 python tools/dense_groups.py 10 >> $O/dense.log 2>&1
done
cat $O/dense.log | cut -c1-250
GPL_DEBUG_TUNE=1 GPL_DEBUG_MODEL=1 timeout 2400 python experiments.py model > $O/model.log 2>&1; cp gpurun_out/model_vs_autotune_sf100.json $O/; tail -c 300 $O/model.log
