"""Run W warm + K query steps (run_query + fetch) — for ncu launch lists (diagnostics)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=torch.cuda.current_stream())
queries.load_database(ctx, ddb, borrow=True)
text = queries.plan_text(q, db)
for i in range(3 + steps):
    if i == 3:  # pinned options (e.g. consumer_warps=16,packets=2) after λ and the profile exist
        for kv in filter(None, os.environ.get("GPL_OPTS", "").split(",")):
            k, v = kv.split("=")
            ctx.set_option(k, int(v))
    ctx.run_query(text)
    r = ctx.fetch_result()
print(q, sf, r.stats["kernel_ms"], r.stats["op_pass"])
