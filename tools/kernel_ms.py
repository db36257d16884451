"""Per-query probe-kernel and step times at one scale factor (the model's shapes, or gpl_autotune's with
GPL_AUTOTUNE=1): median over 20 graph-replayed steps with L2 flushed, CUDA events on the library's stream.
usage: [GPL_OPTS=k=v,...] [GPL_AUTOTUNE=1|builds] python tools/kernel_ms.py SF Q5 Q7 ..."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

sf = float(sys.argv[1])
qs = sys.argv[2:] or ["Q5"]
need = sorted(set().union(*[set(queries.TABLES[q]) for q in qs]) | {"region", "nation"})
db = tpchgen.generate(sf, tables=need)
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
stream = torch.cuda.current_stream()
flush = torch.empty(2 * torch.cuda.get_device_properties(dev).L2_cache_size, dtype=torch.uint8, device=dev)
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for q in qs:
    ctx = gpl.Context(0, stream=stream)
    queries.load_database(ctx, db, queries.TABLES[q])
    text = queries.plan_text(q, db, (19981101,) if q == "L1" else None)  # L1: the non-empty 1998 variant (R1)
    for kv in filter(None, os.environ.get("GPL_OPTS", "").split(",")):  # e.g. GPL_OPTS=nibble_cells=0
        key, v = kv.split("=")
        ctx.set_option(key, int(v))
    mode = os.environ.get("GPL_AUTOTUNE", "0")  # 1: builds + probe measured; builds: the builds only
    if mode in ("1", "builds"):
        ctx.set_option("autotune_probe", 0 if mode == "builds" else 1)
        ctx.autotune(text)
    for _ in range(8):
        ctx.run_query(text)
        r = ctx.fetch_result()
    ks, ss = [], []
    for _ in range(20):
        flush.zero_()
        ev0.record(stream)
        ctx.run_query(text)
        ev1.record(stream)
        r = ctx.fetch_result()
        ks.append(r.stats["kernel_ms"])
        ss.append(ev0.elapsed_time(ev1))
    k, st = statistics.median(ks), statistics.median(ss)
    b = r.stats["bytes_scanned"]
    print(f"{q} SF {sf}: step {st:.4f} ms, kernel {k:.4f} ms, own {b / 1e9:.3f} GB = {b / k / 1e6:.0f} GB/s "
          f"({b / k / 1e6 / 6544:.3f}), shape {r.stats['stage_rows']}x{r.stats['ring_depth']} "
          f"W{r.stats['consumer_warps']} grid {r.stats['grid']} pk {r.stats['packets']} dr {r.stats['drain_warps']}", flush=True)
    ctx.close()
