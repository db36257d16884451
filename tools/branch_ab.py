"""A/B of the whole-query graph with independent build segments on two capture lanes (graph_branches
1) vs one lane (0): step time (graph replay, L2 flushed, CUDA events), results identical.
usage: python tools/branch_ab.py Q5 1.0"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
stream = torch.cuda.current_stream()
ddb = type("D", (), {})()
ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=stream)
queries.load_database(ctx, ddb, borrow=True)
text = queries.plan_text(q, db)
ctx.autotune(text)
flush = torch.empty(2 * torch.cuda.get_device_properties(dev).L2_cache_size, dtype=torch.uint8, device=dev)
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
res = {}
for br in (0, 1, 0, 1):
    ctx._lib.gpl_set_option(ctx._h, b"graph_branches", br)  # keeps the autotuned shapes
    for _ in range(6):
        ctx.run_query(text)
        r = ctx.fetch_result()
    ts = []
    for _ in range(30):
        flush.zero_()
        ev0.record(stream)
        ctx.run_query(text)
        ev1.record(stream)
        r = ctx.fetch_result()
        ts.append(ev0.elapsed_time(ev1))
    res.setdefault(br, []).append(statistics.median(ts))
    key = (tuple(r.keys), tuple(tuple(a) for a in r.aggs))
    res.setdefault("keys", set()).add(key)
print(f"{q} SF {sf}: one lane {res[0]} ms, two lanes {res[1]} ms, results identical: {len(res['keys']) == 1}")
