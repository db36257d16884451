"""Per-call host/device timing of one bench step (diagnostics)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))  # a real stream shared with libgpl
stream = torch.cuda.current_stream()
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=stream)
queries.load_database(ctx, ddb, borrow=False)
segs = queries.segments(queries.plan_text(q, db))
for _ in range(5):
    for s in segs[:-1]: ctx.build_hash(s)
    ctx.run_plan(segs[-1]); ctx.fetch_result()
evs = [torch.cuda.Event(enable_timing=True) for _ in range(len(segs) + 2)]
torch.cuda.synchronize()
host = []
for it in range(3):
    t0 = time.perf_counter(); evs[0].record(stream)
    hs = []
    for i, s in enumerate(segs[:-1]):
        a = time.perf_counter(); ctx.build_hash(s); hs.append(time.perf_counter() - a); evs[i + 1].record(stream)
    a = time.perf_counter(); ctx.run_plan(segs[-1]); hs.append(time.perf_counter() - a); evs[len(segs)].record(stream)
    a = time.perf_counter(); r = ctx.fetch_result(); hs.append(time.perf_counter() - a); evs[-1].record(stream)
    torch.cuda.synchronize()
    tot = time.perf_counter() - t0
    dev_ms = [evs[i].elapsed_time(evs[i + 1]) for i in range(len(evs) - 1)]
    print(f"iter {it}: host total {tot*1e3:.3f} ms; host per call (ms) {[round(h*1e3,3) for h in hs]}; "
          f"device per segment (ms) {[round(x,3) for x in dev_ms]}; kernel {r.stats['kernel_ms']:.3f}")
# host-only overheads with the GPU idle
torch.cuda.synchronize()
import timeit
n = 200
t = timeit.timeit(lambda: ctx.fetch_result(), number=n) / n
print(f"fetch_result with idle GPU: {t*1e6:.1f} us")
t = timeit.timeit(lambda: ctx._lib.gpl_sync(ctx._h), number=n) / n
print(f"gpl_sync (idle): {t*1e6:.1f} us")
text = queries.plan_text(q, db)
ctx.run_query(text); ctx.fetch_result(); ctx.run_query(text); ctx.fetch_result()
torch.cuda.synchronize()
t0 = time.perf_counter(); ctx.run_query(text); t1 = time.perf_counter(); r = ctx.fetch_result(); t2 = time.perf_counter()
print(f"run_query (graph replay) host {1e6*(t1-t0):.1f} us; fetch (incl. wait) {1e6*(t2-t1):.1f} us; kernel {r.stats['kernel_ms']*1e3:.1f} us")
evs = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
for i in range(3):
    evs[0].record(); ctx.run_query(text); evs[1].record(); r = ctx.fetch_result(); evs[2].record(); torch.cuda.synchronize()
    print(f"device: graph {evs[0].elapsed_time(evs[1])*1e3:.1f} us, to-fetch-end {evs[1].elapsed_time(evs[2])*1e3:.1f} us")
