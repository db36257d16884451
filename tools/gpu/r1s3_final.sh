# session-3 final: full GPU suite, smoke, default bench, launch list, SF100 + SF10 benches, Q3 verification
mkdir -p gpurun_out/final2; make -j16 > gpurun_out/make.log 2>&1; echo "make rc=$?"
timeout -s KILL 1500 python -m pytest tests -m gpu -q > gpurun_out/final2/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/final2/pytest_gpu.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final2/smoke.log 2>&1; echo "smoke rc=$?"; tail -4 gpurun_out/final2/smoke.log
timeout -s KILL 600 python bench.py > gpurun_out/final2/bench.json 2> gpurun_out/final2/bench.err; echo "bench rc=$?"; cat gpurun_out/final2/bench.json
timeout -s KILL 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/final2/bench_ref.json 2>/dev/null; echo "ref rc=$?"; cat gpurun_out/final2/bench_ref.json
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final2/launches_q5_sf1.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu-list rc=$?"
for q in Q14 Q5 Q7 Q8 Q9 Q3; do
  timeout -s KILL 900 python bench.py --query $q --sf 100 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/final2/${q}_sf100.json 2>/dev/null; echo "$q rc=$?"
done
timeout -s KILL 600 python bench.py --query Q9 --sf 10 --steps 10 > gpurun_out/final2/Q9_sf10.json 2>/dev/null; echo "Q9 sf10 rc=$?"
timeout -s KILL 600 python bench.py --query Q3 --sf 10 --steps 10 --no-cpu-baseline > gpurun_out/final2/Q3_sf10.json 2>/dev/null; echo "Q3 sf10 rc=$?"
