"""Kernel time of a dense shared-memory group-by (AGG_SMEM, ~all rows into 11 groups) at SF S:
the case SURVEY A7's warp pre-reduction is for. usage: python tools/dense_groups.py [sf] [libgpl.so]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

sf = float(sys.argv[1]) if len(sys.argv) > 1 else 10.0
if len(sys.argv) > 2:
    gpl.LIB_PATH = os.path.abspath(sys.argv[2])
PLAN = """run lineitem
filter l_shipdate <= 19981101
group l_discount 0 11
value l_extendedprice * (100 - l_discount) - l_extendedprice * (400 + l_tax)
agg count
agg sum"""
db = tpchgen.generate(sf, tables=["lineitem"])
ctx = gpl.Context(0)
queries.load_database(ctx, db, ["lineitem"])
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ts = []
for i in range(12):
    flush.zero_()
    torch.cuda.synchronize()
    ctx.run_query(PLAN)
    r = ctx.fetch_result()
    if i >= 4:
        ts.append(r.stats["kernel_ms"])
ms = statistics.median(ts)
print(json.dumps({"lib": gpl.LIB_PATH, "sf": sf, "rows": db.nrows("lineitem"), "kernel_ms": ms,
                  "agg_mode": r.stats["agg_mode"], "bytes": r.stats["bytes_scanned"],
                  "own_gbs": r.stats["bytes_scanned"] / ms / 1e6, "sum_g0": str(r.aggs[0][1])}))
