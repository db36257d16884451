"""Fold an ncu --csv launch list (--metrics ...) into one line per kernel launch."""
import csv
import sys
from collections import OrderedDict

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"]
if not hi:
    print("no ncu rows in", sys.argv[1])
    sys.exit(0)
hdr = rows[hi[0]]
ki, mi, vi, ii = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
ks = OrderedDict()
for r in rows[hi[0] + 1:]:
    if len(r) > vi:
        ks.setdefault(r[ii], {"name": r[ki]})[r[mi]] = r[vi].replace(",", "")
tot = 0.0
for k, v in ks.items():
    t = float(v.get("gpu__time_duration.sum", 0)) / 1e3
    tot += t
    extra = " ".join(f"{m.split('__')[1].split('.')[0]}={v[m]}" for m in v if m not in ("name", "gpu__time_duration.sum"))
    print(f"  {k:>3} {v['name'][:40]:40s} {t:9.1f} us  {extra}")
print(f"  total {tot:.1f} us")
