make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 600 python -m pytest tests -m gpu -x -q -k "gamma or autotune or profiled or schedule" > gpurun_out/pytest_gpu_d.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu_d.log
timeout -s KILL 900 python experiments.py gamma > gpurun_out/gamma.log 2>&1; echo "gamma rc=$?"; tail -c 3000 gpurun_out/gamma.log
timeout -s KILL 600 python experiments.py warps > gpurun_out/warps.log 2>&1; echo "warps rc=$?"; tail -c 1500 gpurun_out/warps.log
python - <<'PY'
import json
d=json.load(open('gpurun_out/warp_sweep.json'))
for p in d['points']: print(p)
d=json.load(open('gpurun_out/gamma_calibration.json'))
for k,v in d['curves'].items(): print(k, [round(x['gbs']) for x in v], round(v[0]['t0_us'],1))
for s in d['sweeps']:
  print(s['sf'], s['gamma_calibrated'], [(p['tile_rows'], round(p['measured_ms'],4), round(p['predicted_ms'],4)) for p in s['points']])
PY
