"""A/B of a build segment's probe split: every probe in the stage phase (insert straight from the staged
tile) vs the probes in the queue phase (`split 0`: the filters' survivors are queued, the drain probes
and inserts; a dense build zero-fills in the stage phase). Whole-query step (graph replay, L2 flushed,
CUDA events) and the build alone, results identical.
usage: python tools/build_split_ab.py Q5 100 HT_O [autotune 0|1]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
ht = sys.argv[3] if len(sys.argv) > 3 else "HT_O"
tune = len(sys.argv) > 4 and sys.argv[4] == "1"
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
stream = torch.cuda.current_stream()
ctx = gpl.Context(0, stream=stream)
queries.load_database(ctx, db)
base = queries.plan_text(q, db)
segs = queries.segments(base)


def with_split(sp):
    alt = []
    for s in segs:
        if f"\nbuild {ht}\n" in "\n" + s:
            s = s.rstrip("\n") + f"\nsplit {sp}\n"
        alt.append(s if s.endswith("\n") else s + "\n")
    return "".join(alt)


variants = {"model": base, "stage": with_split(4), "queue": with_split(0)}
bseg = {k: [s for s in queries.segments(t) if f"build {ht}\n" in s][0] for k, t in variants.items()}
flush = torch.empty(2 * torch.cuda.get_device_properties(dev).L2_cache_size, dtype=torch.uint8, device=dev)
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
out = {}
keys = set()
for rnd in range(2):
    for name, text in variants.items():
        ctx.close()
        ctx = gpl.Context(0, stream=stream)
        queries.load_database(ctx, db)
        if tune:
            ctx.autotune(text)
        for _ in range(6):
            ctx.run_query(text)
            r = ctx.fetch_result()
        ts = []
        for _ in range(20):
            flush.zero_()
            ev0.record(stream)
            ctx.run_query(text)
            ev1.record(stream)
            r = ctx.fetch_result()
            ts.append(ev0.elapsed_time(ev1))
        bs = []
        for _ in range(8):
            flush.zero_()
            ev0.record(stream)
            ctx.build_hash(bseg[name])
            ev1.record(stream)
            torch.cuda.synchronize()
            bs.append(ev0.elapsed_time(ev1))
        out.setdefault(name, []).append((round(statistics.median(ts), 4), round(statistics.median(bs), 4)))
        keys.add((tuple(r.keys), tuple(tuple(a) for a in r.aggs)))
print(f"{q} SF {sf} {ht} (step ms, build ms) autotune={tune}: {out}; results identical: {len(keys) == 1}")
