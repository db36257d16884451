# config 4 (1 GPU): every paper query at SF 100 through bench.py, + config 3 (Q9 SF 10)
make -j16 > gpurun_out/make.log 2>&1
mkdir -p gpurun_out/sf100
for q in Q14 Q5 Q7 Q8 Q9; do
  timeout 900 python bench.py --query $q --sf 100 --steps 10 --warmup 3 > gpurun_out/sf100/$q.json 2> gpurun_out/sf100/$q.err
  echo "$q rc=$?"; tail -c 600 gpurun_out/sf100/$q.json
done
timeout 600 python bench.py --query Q9 --sf 10 > gpurun_out/sf100/Q9_sf10.json 2> gpurun_out/sf100/Q9_sf10.err
timeout 1500 python tools/verify_sf100.py gpurun_out/verify_sf100_r01b.json 100 > gpurun_out/verify.log 2>&1; echo "verify rc=$?"
