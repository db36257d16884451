"""A small run of every plan (paper queries + Q3's hash group-by with and without LIMIT) for
compute-sanitizer (memcheck / racecheck / synccheck): eager runs and graph replays, bit-exact vs oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

db = tpchgen.generate(0.02, seed=3)
ctx = gpl.Context(0)
queries.load_database(ctx, db)
ok = True
for q in queries.QUERIES + queries.EXTRA_QUERIES:
    params = (19981101,) if q == "L1" else None
    o = oracle.run(q, db, params)
    if q == "Q3":
        o_all, o = o, oracle.order_limit("Q3", o)
    for _ in range(3):
        r = queries.run_query(ctx, q, db, params)
        ok &= r.keys == o.keys and r.aggs == o.aggs
    print(q, "exact" if ok else "MISMATCH", flush=True)
full = "\n".join(ln for ln in queries.plan_text("Q3", db).splitlines() if not ln.startswith(("order", "limit")))
for _ in range(3):
    ctx.run_query(full)
    r = ctx.fetch_result()
ok &= r.keys == o_all.keys and r.aggs == o_all.aggs
print("Q3 all groups", "exact" if ok else "MISMATCH")
sys.exit(0 if ok else 1)
