"""Kernel time of one query at a pinned pipeline shape (diagnostics): python tools/pin_shape.py Q7 100 S D W k np tile"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

q, sf = sys.argv[1], float(sys.argv[2])
S, D, W, k, npk, tile = (int(x) for x in sys.argv[3:9])
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
ddb = type("D", (), {})()
ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=torch.cuda.current_stream())
queries.load_database(ctx, ddb, borrow=True)
text = queries.plan_text(q, db)
flush = torch.empty(2 * torch.cuda.get_device_properties(dev).L2_cache_size, dtype=torch.uint8, device=dev)
for _ in range(3):  # λ and the model's profile first (unpinned)
    ctx.run_query(text)
    ctx.fetch_result()
for name, v in (("stage_rows", S), ("ring_depth", D), ("consumer_warps", W), ("ctas_per_sm", k), ("packets", npk),
                ("probe_split", 1)):
    ctx.set_option(name, v)
for kv in filter(None, os.environ.get("GPL_OPTS", "").split(",")):  # e.g. lazy_columns=0,clustered=0
    name, v = kv.split("=")
    ctx.set_option(name, int(v))
ts = []
for i in range(8):
    flush.zero_()
    ctx.run_query(text, tile)
    r = ctx.fetch_result()
    if i >= 3:
        ts.append(r.stats["kernel_ms"])
print(f"{q} SF {sf} S {S} D {D} W {W} k {k} np {npk} tile {tile}: kernel {statistics.median(ts):.4f} ms "
      f"(lazy {r.stats['lazy_columns']}, split {r.stats['probe_split']}, tile used {r.stats['tile_rows_used']})")
