"""Time each build segment of a query under pipeline shapes (diagnostics)."""
import sys, os, statistics, itertools
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 5.0
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
stream = torch.cuda.current_stream()
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=stream)
queries.load_database(ctx, ddb, borrow=True)
segs = queries.segments(queries.plan_text(q, db))
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
def time_builds(reps=5):
    out = []
    for s in segs[:-1]:
        ts = []
        for i in range(reps + 1):
            flush.zero_()
            ev[0].record(stream); ctx.build_hash(s); ev[1].record(stream); ev[1].synchronize()
            if i: ts.append(ev[0].elapsed_time(ev[1]) * 1e3)
        out.append(round(statistics.median(ts), 1))
    ctx.run_plan(segs[-1]); ctx.fetch_result()
    return out
names = [s.split()[1] for s in segs[:-1]]
print(q, sf, "builds", names)
ctx.set_option("build_pipeline", 0); print("build kernels            ", time_builds())
ctx.set_option("build_pipeline", 1); print("pipeline (model)         ", time_builds())
for S, Dp, W, k, sp in itertools.product([512, 1024, 2048], [3, 4], [4, 8], [1, 2], [-2, 1]):
    try:
        for key, v in (("stage_rows", S), ("ring_depth", Dp), ("consumer_warps", W), ("ctas_per_sm", k), ("probe_split", sp)):
            ctx.set_option(key, v)
        print(f"S={S:5d} D={Dp} W={W:2d} k={k} split={sp:2d} ", time_builds(3), flush=True)
    except gpl.GplError as e:
        print(f"S={S} D={Dp} W={W} k={k} split={sp}: {e}")
