"""A small run of every plan and every kernel variant for compute-sanitizer (memcheck / racecheck /
synccheck), bit-exact vs the oracle: the paper plans (clustered probe, late materialisation with
gathers at first use, register drain fields), Q3's hash group-by (device top-k and the full device sort),
QF's fan-out join (multi build, chained probe), operator-specialised drain warps D = 1 and 2, forced
global int128 accumulators, a dense shared-memory group-by (lane-private copies), builds with queue-phase
probes and inserts, 4-bit cells (dense, atomic, random key gaps), and the KBE / GPL (w/o CE) baselines.
Eager runs and graph replays, SF 0.02."""
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


def expect(q, params=None):
    o = oracle.run("Q5" if q == "Q5P" else q, db, params)  # Q5P: Q5 through a partitioned hash join
    return oracle.order_limit("Q3", o) if q == "Q3" else oracle.finalize("Q5" if q == "Q5P" else q, o)


def check(tag, q, params=None, kbe=False, reps=3):
    global ok
    o = expect(q, params)
    for _ in range(reps):
        r = queries.run_query(ctx, q, db, params, kbe=kbe)
        good = r.keys == o.keys and r.aggs == o.aggs
        ok &= good
    print(tag, q, "exact" if good else "MISMATCH", flush=True)


plans = queries.QUERIES + queries.EXTRA_QUERIES
P = {"L1": (19981101,)}
for q in plans:
    check("default", q, P.get(q))
for nd in (1, 2):
    ctx.set_option("drain_warps", nd)
    ctx.set_option("consumer_warps", 6)
    for q in ("Q5", "Q7", "Q3", "QF"):
        check(f"drain_warps={nd}", q, P.get(q))
ctx.set_option("drain_warps", -1)
ctx.set_option("consumer_warps", -1)
ctx.set_option("lazy_columns", 1)
for q in ("Q5", "Q9", "Q14"):
    check("lazy=1", q, P.get(q))
ctx.set_option("lazy_columns", -1)
ctx.set_option("agg_mode", 2)
for q in ("Q5", "Q9"):
    check("agg_global", q, P.get(q))
ctx.set_option("agg_mode", -1)
for q in ("Q5", "Q9"):
    check("kbe", q, P.get(q), kbe=True, reps=1)
ctx.set_option("kbe_tile_rows", 3000)
for q in ("Q5", "Q9"):
    check("gpl_wo_ce", q, P.get(q), kbe=True, reps=1)
ctx.set_option("kbe_tile_rows", 0)
# Q3 without LIMIT: every group, full device sort (ORDER BY revenue desc, o_orderdate)
o_all = oracle.run("Q3", db)
want = sorted(zip(o_all.keys, o_all.aggs), key=lambda ka: (-ka[1][1], ka[0][1], ka[0]))
text = "\n".join(ln for ln in queries.plan_text("Q3", db).splitlines() if not ln.startswith("limit"))
for _ in range(3):
    ctx.run_query(text)
    try:
        r = ctx.fetch_result()
    except gpl.GplError:
        continue
good = list(zip(r.keys, r.aggs)) == want
ok &= good
print("Q3 full device sort", "exact" if good else "MISMATCH")
# dense shared-memory group-by: lane-private table copies, every row adding (exact Python-int sums)
L = db.tables["lineitem"]
want = {}
for g, ep, q_, t in zip(L["l_discount"].tolist(), L["l_extendedprice"].tolist(), L["l_quantity"].tolist(),
                        L["l_tax"].tolist()):
    c, v = want.get(g, (0, 0))
    want[g] = (c + 1, v + ep * (100 - g) - ep * q_ * (40 + t))
dense = """run lineitem
group l_discount 0 11
value l_extendedprice * (100 - l_discount) - l_extendedprice * l_quantity * (40 + l_tax)
agg count
agg sum"""
for _ in range(3):
    ctx.run_query(dense)
    r = ctx.fetch_result()
good = r.stats["agg_mode"] == 1 and {k[0]: tuple(a) for k, a in zip(r.keys, r.aggs)} == want
ok &= good
print("dense smem groups", "exact" if good else "MISMATCH")
# builds with their probes and insert in the queue phase (a dense build zero-fills in the stage phase,
# the drain writes the cells), and 4-bit cells (dense: whole-byte stores + atomics on shared bytes;
# atomic builds; clustered and global probes)
ctx.set_option("probe_split", 0)
for q in ("Q5", "Q8"):
    check("build_split=0", q, P.get(q))
ctx.set_option("probe_split", -2)
ctx.set_option("nibble_cells", 1)
for q in ("Q5", "Q7", "Q9"):
    check("nibble", q, P.get(q))
ctx.set_option("dense_build", 0)
check("nibble atomic", "Q7")
ctx.set_option("dense_build", 1)
import numpy as np  # noqa: E402
rng = np.random.default_rng(5)
k = (np.cumsum(rng.integers(1, 4, 20001)) + 1000).astype(np.int32)
pay = rng.integers(3, 17, k.size).astype(np.int32)
f = rng.integers(0, 100, k.size).astype(np.int32)
ctx.load_columns("nt_dim", {"k": k, "p": pay, "f": f})
ctx.load_columns("nt_fact", {"x": np.arange(int(k[0]) - 5, int(k[-1]) + 6, dtype=np.int32)})
plan = ("build NT\nscan nt_dim\nfilter f < 60\nkey k\npayload p\n\n"
        "run nt_fact\nprobe NT x -> pv\ngroup pv 3 17\nagg count\n")
vals, cnts = np.unique(pay[f < 60], return_counts=True)
for _ in range(3):
    ctx.run_query(plan)
    r = ctx.fetch_result()
good = r.keys == [(int(v),) for v in vals] and r.aggs == [[int(c)] for c in cnts]
ok &= good
print("nibble random gaps", "exact" if good else "MISMATCH")
ctx.set_option("nibble_cells", 0)
sys.exit(0 if ok else 1)
