"""Measure the fused kernel over pipeline shapes (stage rows x depth x warps) — diagnostics."""
import sys, os, itertools, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))  # a real stream shared with libgpl
stream = torch.cuda.current_stream()
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=stream)
queries.load_database(ctx, ddb)
segs = queries.segments(queries.plan_text(q, db))
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
def run(n=6):
    ts = []
    for i in range(n):
        for s in segs[:-1]: ctx.build_hash(s)
        flush.zero_()
        ctx.run_plan(segs[-1]); r = ctx.fetch_result()
        if i >= 2: ts.append(r.stats["kernel_ms"])
    return statistics.median(ts), r
base, r = run()
print(f"{q} SF{sf} auto: {base*1e3:.1f} us  cfg={ {k: r.stats[k] for k in ('stage_rows','ring_depth','consumer_warps','tile_rows_used','probe_split')} }  GB/s={r.stats['bytes_scanned']/base/1e6:.0f}")
best = (base, "auto")
for S, Dp, W in itertools.product([512, 1024, 2048, 4096], [2, 3, 4, 6, 8], [4, 8, 12, 16]):
    try:
        ctx.set_option("stage_rows", S); ctx.set_option("ring_depth", Dp); ctx.set_option("consumer_warps", W)
        t, r = run(5)
    except gpl.GplError:
        continue
    tag = f"S={S} D={Dp} W={W}"
    if t < best[0]: best = (t, tag)
    print(f"  {tag:22s} {t*1e3:7.1f} us  {r.stats['bytes_scanned']/t/1e6:6.0f} GB/s")
print("best", best)
