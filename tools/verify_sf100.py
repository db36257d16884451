"""SF 100 verification on one B200 (BASELINE config 4 sizes), written to a JSON record.

For every query:
  * full  = the fused pipeline over the whole SF 100 database (600M lineitem rows);
  * additivity: the same query over 4 order-key shards, int128 partials merged
    with gpl_merge_partials, must equal `full` exactly (the multi-GPU layout);
  * sampled parity: shard 0 of 200 (≈3M lineitem rows with the FULL SF 100
    dimension tables) on the GPU must equal the CPU oracle exactly.

usage: python tools/verify_sf100.py [out.json] [sf]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "verify_sf100.json")
SF = float(sys.argv[2]) if len(sys.argv) > 2 else 100.0
QS = ["Q14", "Q5", "Q7", "Q8", "Q9", "L1"]
PARAMS = {"L1": (19981101,)}
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
ctx = gpl.Context(0, stream=torch.cuda.current_stream())
record = {"sf": SF, "queries": {}}


def run(db, q):
    queries.load_database(ctx, db)
    return queries.run_query(ctx, q, db, PARAMS.get(q))


t0 = time.time()
full = tpchgen.generate(SF)
record["gen_full_s"] = time.time() - t0
record["lineitem_rows"] = full.nrows("lineitem")
res_full = {}
for q in QS:
    r = run(full, q)
    res_full[q] = r
    record["queries"][q] = {"groups": len(r.keys), "count": sum(a[0] for a in r.aggs), "kernel_ms": r.stats["kernel_ms"]}
del full

W = 4
parts = {q: [] for q in QS}
for rk in range(W):
    shard = tpchgen.generate(SF, rank=rk, world=W)
    for q in QS:
        run(shard, q)
        parts[q].append(ctx.fetch_partials())
    del shard
for q in QS:
    merged = gpl.merge_partials(np.concatenate(parts[q]), W)
    # the partial layout depends only on the plan text (same at every SF):
    # run q once on a tiny database so the context decodes with q's layout
    tiny = tpchgen.generate(0.01)
    run(tiny, q)
    dec = queries.decode_keys(q, ctx.decode_partials(merged), tiny)
    ok = dec.keys == res_full[q].keys and dec.aggs == res_full[q].aggs
    record["queries"][q]["additivity_4_shards"] = bool(ok)

sample = tpchgen.generate(SF, rank=0, world=200)
for q in QS:
    t = time.time()
    o = oracle.run(q, sample, PARAMS.get(q))
    ot = time.time() - t
    r = run(sample, q)
    record["queries"][q]["sample_rows"] = sample.nrows("lineitem")
    record["queries"][q]["sample_parity"] = bool(r.keys == o.keys and r.aggs == o.aggs)
    record["queries"][q]["oracle_sample_s"] = ot
record["all_ok"] = all(v["additivity_4_shards"] and v["sample_parity"] for v in record["queries"].values())
json.dump(record, open(out, "w"), indent=1)
print(json.dumps(record))
