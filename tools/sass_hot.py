"""Summarise an `ncu --page source --csv --print-source sass` export: for one kernel section (default: the
last, i.e. the probe kernel of a query step), the total instructions executed and the hottest SASS lines by
stall samples. usage: python tools/sass_hot.py file.csv [section] [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
starts = [i for i, r in enumerate(rows) if r and r[0] == "Kernel Name"]
sec = int(sys.argv[2]) if len(sys.argv) > 2 else len(starts) - 1
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
st = starts[sec]
end = starts[sec + 1] if sec + 1 < len(starts) else len(rows)
hdr = rows[st + 1]
body = [r for r in rows[st + 2:end] if len(r) == len(hdr)]
ie, src, samp = hdr.index("Instructions Executed"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
tot = sum(int(r[ie].replace(",", "") or 0) for r in body)
tots = sum(int(r[samp].replace(",", "") or 0) for r in body)
print(f"section {sec}: {len(body)} SASS lines, {tot} warp instructions executed, {tots} stall samples")
agg = {}
for r in body:
    for h in stalls:
        agg[h] = agg.get(h, 0) + int(r[hdr.index(h)].replace(",", "") or 0)
print("stall totals:", ", ".join(f"{k[6:]}={v}" for k, v in sorted(agg.items(), key=lambda kv: -kv[1])[:8]))
for r in sorted(body, key=lambda r: -int(r[samp].replace(",", "") or 0))[:top]:
    worst = max(stalls, key=lambda h: int(r[hdr.index(h)].replace(",", "") or 0))
    print(f"{int(r[samp].replace(',', '') or 0):7d} {int(r[ie].replace(',', '') or 0):11d} {worst[6:]:14s} {r[src][:90]}")
