#!/bin/bash
# One validation round trip: the whole GPU suite, smoke, the default bench line, and the per-query
# step/kernel medians at SF 100 with the model's shapes (tools/kernel_ms.py), every kernel variant exact.
# usage: bash tools/gpu_check.sh TAG
TAG=${1:-check}
O=gpurun_out/$TAG; mkdir -p $O
make -j16 > $O/make.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log; tail -3 $O/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log; tail -2 $O/smoke.log
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; head -c 400 $O/bench.json; echo
# the multi-rank merge path over NCCL at one rank (torchrun, process group, all-gather, fixed-order merge)
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 \
    bench.py --collective --steps 20 --no-cpu-baseline > $O/bench_collective.json 2> $O/bench_collective.err
python -c "import json; d=[json.loads(l) for l in open('$O/bench_collective.json') if l.startswith('{')][0]; print('collective', d['collective'], d['ms_per_step'], d['kernel_ms'])"
timeout 1500 python tools/kernel_ms.py 100 Q5 Q7 Q8 Q9 Q14 Q3 > $O/kernel_ms.txt 2>&1; grep SF $O/kernel_ms.txt
# every kernel variant bit-exact (the compute-sanitizer driver, run plain: the pool has the sanitizer closed)
timeout 900 python tools/sanitize_run.py > $O/variants.log 2>&1; echo "variants rc=$?" >> $O/variants.log; tail -3 $O/variants.log
