"""Kernel time with late materialisation off / auto / forced, per query (diagnostics)."""
import sys, os, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries
sf = float(sys.argv[1]) if len(sys.argv) > 1 else 20.0
qs = sys.argv[2].split(",") if len(sys.argv) > 2 else ["Q14", "Q5", "Q7", "Q8", "Q9"]
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
db = tpchgen.generate(sf, tables=["part", "partsupp", "supplier", "customer", "orders", "lineitem", "nation", "region"])
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=torch.cuda.current_stream())
queries.load_database(ctx, ddb, borrow=True)
for q in qs:
    text = queries.plan_text(q, db)
    ref = None
    for mode, cl in ((0, 0), (-1, 0), (-1, 1), (0, 1)):
        ctx.set_option("lazy_columns", mode)
        ctx.set_option("clustered", cl)
        ts = []
        for i in range(7):
            flush.zero_(); ctx.run_query(text); r = ctx.fetch_result()
            if i >= 2: ts.append(r.stats["kernel_ms"])
        if ref is None: ref = (r.keys, r.aggs)
        assert (r.keys, r.aggs) == ref
        t = statistics.median(ts)
        st = r.stats
        print(f"{q} SF{sf} lazy={mode:2d} clustered={cl}: kernel {t*1e3:8.1f} us  lazy_cols={st['lazy_columns']} P={st['packets']} split={st['probe_split']} "
              f"bytes {st['bytes_scanned']/1e9:.3f}/{st['bytes_full_scan']/1e9:.3f} GB -> {st['bytes_scanned']/t/1e6:.0f} GB/s "
              f"(full-scan equiv {st['bytes_full_scan']/t/1e6:.0f} GB/s)", flush=True)
    ctx.set_option("lazy_columns", -1)
    ctx.set_option("clustered", 1)
