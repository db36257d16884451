"""Q3 (NEXT-4: hash group-by + device ORDER BY/LIMIT) at SF 100 on one B200, written to a JSON record.

  * full: Q3 over the whole database (600M lineitem rows at SF 100) — the top-10 rows and the count of
    distinct groups;
  * shard union: a group key contains l_orderkey and shards are order-key ranges, so the groups of W
    shards are disjoint: the top-10 of the union of the shards' top-10s must equal the full top-10,
    and the shards' distinct-group counts must add up to the full count (the multi-GPU layout);
  * sampled parity: shard 0 of 200 (full dimension tables) on the GPU equals the CPU oracle exactly —
    both the ORDER BY/LIMIT rows and the complete group set (the no-LIMIT plan).

usage: python tools/verify_q3.py [out.json] [sf]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import oracle  # noqa: E402
import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "verify_q3.json")
SF = float(sys.argv[2]) if len(sys.argv) > 2 else 100.0
TABLES = queries.TABLES["Q3"]
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
ctx = gpl.Context(0, stream=torch.cuda.current_stream())
rec = {"sf": SF}


def run(db):
    queries.load_database(ctx, db, TABLES)
    r = None
    for _ in range(3):  # warm: sizes the aggregation table from the groups seen
        r = queries.run_query(ctx, "Q3", db)
    return r


t0 = time.time()
full = tpchgen.generate(SF, tables=TABLES)
rec["gen_full_s"] = time.time() - t0
rec["lineitem_rows"] = full.nrows("lineitem")
rf = run(full)
rec["full"] = {"top10": [list(k) + a for k, a in zip(rf.keys, rf.aggs)], "groups_total": rf.stats["groups_total"],
               "kernel_ms": rf.stats["kernel_ms"], "hash_slots": rf.stats["hash_slots"]}
del full

W = 4
rows, groups = [], 0
for rk in range(W):
    shard = tpchgen.generate(SF, rank=rk, world=W, tables=TABLES)
    r = run(shard)
    rows += list(zip(r.keys, r.aggs))
    groups += r.stats["groups_total"]
    del shard
union = oracle.order_limit("Q3", oracle.Result("Q3", [k for k, _ in rows], [a for _, a in rows]))
rec["shard_union_top10_equal"] = union.keys == rf.keys and union.aggs == rf.aggs
rec["shard_groups_add_up"] = groups == rf.stats["groups_total"]

sample = tpchgen.generate(SF, rank=0, world=200, tables=TABLES)
t = time.time()
o = oracle.run("Q3", sample)
rec["oracle_sample_s"] = time.time() - t
r = run(sample)
want = oracle.order_limit("Q3", o)
rec["sample_rows"] = sample.nrows("lineitem")
rec["sample_groups"] = len(o.keys)
rec["sample_top10_parity"] = r.keys == want.keys and r.aggs == want.aggs
full_plan = "\n".join(ln for ln in queries.plan_text("Q3", sample).splitlines() if not ln.startswith(("order", "limit")))
for _ in range(2):
    ctx.run_query(full_plan)
    try:
        g = ctx.fetch_result()
        break
    except gpl.GplError:
        continue
rec["sample_all_groups_parity"] = g.keys == o.keys and g.aggs == o.aggs
rec["all_ok"] = bool(rec["shard_union_top10_equal"] and rec["shard_groups_add_up"] and rec["sample_top10_parity"]
                     and rec["sample_all_groups_parity"])
with open(out, "w") as f:
    json.dump(rec, f, indent=1)
print(json.dumps({k: v for k, v in rec.items() if k != "full"}))
