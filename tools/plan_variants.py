"""Compare probe orders / shapes for a query at a given SF (diagnostics)."""
import sys, os, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries

q = sys.argv[1]; sf = float(sys.argv[2])
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
stream = torch.cuda.current_stream()
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=stream)
queries.load_database(ctx, ddb)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
base = queries.plan_text(q, db)
variants = {"as-written": base}
lines = base.splitlines()
probes = [i for i, l in enumerate(lines) if l.startswith(("probe ", "semi ", "mark ")) and i > max(j for j, x in enumerate(lines) if x.startswith("run "))]
if len(probes) >= 2:
    rev = list(lines)
    ps = [lines[i] for i in probes][::-1]
    for i, l in zip(probes, ps): rev[i] = l
    variants["probes-reversed"] = "\n".join(rev)
for name, text in variants.items():
    segs = queries.segments(text)
    for split in (-2, 0, 1, 2):
        ctx.set_option("probe_split", split)
        ts = []
        try:
            for i in range(6):
                ctx.run_query(text); flush.zero_()
                ctx.run_query(text); r = ctx.fetch_result()
                if i >= 2: ts.append(r.stats["kernel_ms"])
        except gpl.GplError as e:
            print(name, split, "ERR", e); continue
        t = statistics.median(ts)
        print(f"{name:16s} split={split:2d} kernel {t:.3f} ms  {r.stats['bytes_scanned']/t/1e6:.0f} GB/s  cfg S={r.stats['stage_rows']} D={r.stats['ring_depth']} W={r.stats['consumer_warps']} split_used={r.stats['probe_split']} ops={r.stats['op_pass']}")
ctx.set_option("probe_split", -2)
