"""SURVEY §8(d) oracle timing: the CPU oracle (as it stands) on 1 thread and on every host core at SF 1 and
SF 10 for the paper's queries (index builds + scan + merge, generation excluded), with the CPU model.
usage: python tools/oracle_timing.py [out.json] [sf ...]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import tpchgen  # noqa: E402

out = sys.argv[1] if len(sys.argv) > 1 else None
sfs = [float(x) for x in sys.argv[2:]] or [1.0, 10.0]
T = oracle.host_threads()
rows = []
for sf in sfs:
    db = tpchgen.generate(sf)
    n = db.nrows("lineitem")
    for q in ("Q5", "Q7", "Q8", "Q9", "Q14"):
        for threads in sorted({1, T}):
            reps = 3 if sf <= 1 else 1
            ts = [oracle.timed_run(q, db, None, None, threads)[1] for _ in range(reps)]
            t = statistics.median(ts)
            rows.append({"sf": sf, "query": q, "threads": threads, "ms": 1e3 * t, "fact_rows_per_s": n / t})
            print(f"SF {sf} {q} threads {threads}: {1e3 * t:.1f} ms, {n / t:.3g} rows/s", flush=True)
summary = {"what": "CPU oracle timing (SURVEY §8(d)): 1 thread and all host cores, SF <= 10", "cores": T,
           "cpu_model": oracle.cpu_model(), "points": rows}
if out:
    with open(out, "w") as f:
        json.dump(summary, f, indent=1)
