"""Time explicit pipeline shapes for one query (diagnostics): python tools/try_shapes.py Q5 8 S,D,W,k ..."""
import sys, os, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries
q, sf = sys.argv[1], float(sys.argv[2])
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
ctx = gpl.Context(0, stream=torch.cuda.current_stream())
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
queries.load_database(ctx, ddb)
text = queries.plan_text(q, db)
for spec in sys.argv[3:]:
    vals = list(map(int, spec.split(",")))
    S, Dp, W, k = vals[:4]
    npk = vals[4] if len(vals) > 4 else -1
    sp = vals[5] if len(vals) > 5 else -2
    for key, v in (("stage_rows", S), ("ring_depth", Dp), ("consumer_warps", W), ("ctas_per_sm", k),
                   ("packets", npk), ("probe_split", sp)):
        ctx.set_option(key, v)
    ts = []
    try:
        for i in range(7):
            flush.zero_(); ctx.run_query(text); r = ctx.fetch_result()
            if i >= 2: ts.append(r.stats["kernel_ms"])
    except gpl.GplError as e:
        print(spec, "ERR", e); continue
    t = statistics.median(ts)
    print(f"{q} SF{sf} S={S} D={Dp} W={W} k={k} P={npk} split={r.stats['probe_split']}: {t*1e3:.1f} us  {r.stats['bytes_scanned']/t/1e6:.0f} GB/s", flush=True)
