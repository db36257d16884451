"""Kernel time vs SF for a few queries -> fixed overhead (intercept) + streaming rate (slope)."""
import sys, os, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
stream = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
ctx = gpl.Context(0, stream=stream)
for q, params in (("L1", (19981101,)), ("Q14", None), ("Q5", None)):
    pts = []
    for sf in (0.5, 1, 2, 4, 8):
        db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
        class D: pass
        ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
        queries.load_database(ctx, ddb)
        text = queries.plan_text(q, db, params)
        ctx.autotune(text)
        ts = []
        for i in range(6):
            flush.zero_()
            ctx.run_query(text); r = ctx.fetch_result()
            if i >= 2: ts.append(r.stats["kernel_ms"])
        t = statistics.median(ts)
        pts.append((r.stats["bytes_scanned"], t))
        print(f"{q} SF{sf}: {t*1e3:.1f} us, {r.stats['bytes_scanned']/t/1e6:.0f} GB/s  S={r.stats['stage_rows']} D={r.stats['ring_depth']} W={r.stats['consumer_warps']} grid={r.stats['grid']}", flush=True)
    x = np.array([p[0] for p in pts]); y = np.array([p[1] for p in pts])
    b, a = np.polyfit(x, y, 1)
    print(f"{q}: fixed {a*1e3:.1f} us + {1/b/1e6:.0f} GB/s marginal")
