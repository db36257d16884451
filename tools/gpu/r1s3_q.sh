mkdir -p gpurun_out/diag; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:"gpl_pipeline" -s 40 -c 1 -o gpurun_out/diag/prof_q7_sf100 python bench.py --query Q7 --sf 100 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/diag/ncu_q7.log 2>&1; echo "ncu rc=$?"; tail -2 gpurun_out/diag/ncu_q7.log
timeout -s KILL 900 python bench.py --query Q7 --sf 100 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/diag/Q7_again.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/diag/Q7_again.json'));print('again', d['ms_per_step'],d['kernel_ms'],d['pipeline'])"
nvidia-smi --query-gpu=name,memory.total,clocks.max.mem,clocks.max.sm,pcie.link.gen.max --format=csv
