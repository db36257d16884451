"""Host-side cost of the API calls of one warm query step (diagnostics)."""
import sys, os, time, statistics, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import tpchgen
from paper_conf_sigmod_paulhh16_b200 import gpl, queries

q = sys.argv[1] if len(sys.argv) > 1 else "Q5"
sf = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
db = tpchgen.generate(sf, tables=sorted(set(queries.TABLES[q]) | {"region", "nation"}))
dev = torch.device("cuda", 0)
torch.cuda.set_stream(torch.cuda.Stream(device=dev))
stream = torch.cuda.current_stream()
class D: pass
ddb = D(); ddb.tables = {t: {c: torch.from_numpy(a).to(dev) for c, a in cols.items()} for t, cols in db.tables.items()}
ctx = gpl.Context(0, stream=stream)
queries.load_database(ctx, ddb, borrow=True)
text = queries.plan_text(q, db)
for _ in range(5):
    ctx.run_query(text); ctx.fetch_result()
torch.cuda.synchronize()
raw = text.encode()
def t_us(fn, n=200):
    ts = []
    for _ in range(n):
        torch.cuda.synchronize()
        a = time.perf_counter(); fn(); ts.append(time.perf_counter() - a)
    return statistics.median(ts) * 1e6
print(f"ctx.run_query           {t_us(lambda: ctx.run_query(text)):.1f} us")
print(f"lib.gpl_run_query(raw)  {t_us(lambda: ctx._lib.gpl_run_query(ctx._h, raw, 0)):.1f} us")
print(f"lib.gpl_version         {t_us(lambda: ctx._lib.gpl_version()):.1f} us")
print(f"torch.cuda.synchronize  {t_us(lambda: None):.1f} us")
ctx.run_query(text); torch.cuda.synchronize()
print(f"fetch_result (idle)     {t_us(lambda: ctx.fetch_result()):.1f} us")
print(f"gpl_sync (idle)         {t_us(lambda: ctx._lib.gpl_sync(ctx._h)):.1f} us")
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for name, fn in (("step run_query+fetch", lambda: (ctx.run_query(text), ctx.fetch_result())),):
    ms = []
    for _ in range(50):
        torch.cuda.synchronize(); ev0.record(stream); fn(); ev1.record(stream); ev1.synchronize(); ms.append(ev0.elapsed_time(ev1))
    print(f"{name}: device {statistics.median(ms)*1e3:.1f} us; kernel {ctx.fetch_result().stats['kernel_ms']*1e3:.1f} us")
