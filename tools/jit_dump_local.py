"""Dump the plan-specialised kernel source of a query's probe segment on a host-only
context (no GPU): GPL_JIT_DUMP=<dir> python tools/jit_dump_local.py Q [sf] [k=v ...]
then compile it with nvcc (-cubin, sm_100a) to inspect the SASS (diagnostics)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tpchgen  # noqa: E402
from paper_conf_sigmod_paulhh16_b200 import gpl, queries  # noqa: E402

q = sys.argv[1]
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 0.1
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
ctx = gpl.Context(device=-1)
queries.load_database(ctx, db)
segs = queries.segments(queries.plan_text(q, db))
for s in segs[:-1]:
    ctx.build_hash(s)
for kv in sys.argv[3:]:  # options of the probe segment (set after the builds)
    k, v = kv.split("=")
    ctx.set_option(k, int(v))
print(ctx.choose_tile_rows(segs[-1]))
ctx.compile_plan(segs[-1])
