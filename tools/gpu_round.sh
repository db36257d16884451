#!/bin/bash
# One GPU round: parity tests, benches, ncu capture of the fused kernel.
# usage (under gpurun): bash tools/gpu_round.sh TAG [tests|notests]
TAG=${1:-dev}
mkdir -p gpurun_out
if [ "${2:-tests}" = "tests" ]; then
  timeout -s KILL 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
fi
timeout -s KILL 300 python bench.py --no-e2e > gpurun_out/b_q5_sf1_$TAG.json 2> gpurun_out/b_q5_sf1_$TAG.log; cat gpurun_out/b_q5_sf1_$TAG.json
timeout -s KILL 400 python bench.py --query Q9 --sf 10 --steps 10 --no-e2e --no-cpu-baseline > gpurun_out/b_q9_sf10_$TAG.json 2> gpurun_out/b_q9_sf10_$TAG.log; cat gpurun_out/b_q9_sf10_$TAG.json
timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:pipeline -s 3 -c 1 -o gpurun_out/prof_q5_sf1_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1; tail -1 gpurun_out/ncu_$TAG.log
