mkdir -p gpurun_out/diag; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 900 python -m pytest tests -m gpu -q -k "graph" > gpurun_out/pytest_gpu_o.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_o.log
timeout -s KILL 600 python tools/pin_shape.py Q7 100 2048 2 8 2 2 65536; timeout -s KILL 600 python tools/pin_shape.py Q7 100 4096 3 8 1 1 8192
timeout -s KILL 600 python tools/branch_ab.py Q5 1.0; timeout -s KILL 600 python tools/branch_ab.py Q9 10.0
GPL_DEBUG_TUNE=1 timeout -s KILL 900 python bench.py --query Q7 --sf 100 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/diag/Q7.json 2> gpurun_out/diag/Q7.err; echo "Q7 rc=$?"; python -c "import json;d=json.load(open('gpurun_out/diag/Q7.json'));print(d['ms_per_step'],d['kernel_ms'],d['pipeline'])"; grep "autotune: split" gpurun_out/diag/Q7.err | sort -t: -k3 -n | head -8
