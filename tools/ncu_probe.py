"""One warm query step inside a cudaProfilerStart/Stop window (ncu --profile-from-start off):
the launches of exactly one graph-replayed step (clear, builds, fused probe kernel, copy-out).

usage: python tools/ncu_probe.py Q [sf]   (GPL_OPTS="k=v,..." pins options after the warm-up)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 100.0
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
ctx = gpl.Context(0, stream=torch.cuda.current_stream())
queries.load_database(ctx, db)
text = queries.plan_text(q, db)
if os.environ.get("GPL_AUTOTUNE", "1") == "1":
    ctx.autotune(text)
for kv in filter(None, os.environ.get("GPL_OPTS", "").split(",")):
    k, v = kv.split("=")
    ctx.set_option(k, int(v))
for _ in range(6):
    ctx.run_query(text)
    r = ctx.fetch_result()
torch.cuda.synchronize()
torch.cuda.profiler.start()
ctx.run_query(text)
r = ctx.fetch_result()
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print(q, sf, "kernel_ms", r.stats["kernel_ms"], "bytes", r.stats["bytes_scanned"], "op_pass", r.stats["op_pass"],
      {k: r.stats[k] for k in ("stage_rows", "ring_depth", "consumer_warps", "grid", "probe_split", "packets",
                               "lazy_columns", "tile_rows_used")})
