import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]; data = rows[2:]
ia = hdr.index("Instructions Executed"); ss = hdr.index("Warp Stall Sampling (All Samples)")
tot_i = sum(int(r[ia] or 0) for r in data); tot_s = sum(int(r[ss] or 0) for r in data)
print("total warp instr", tot_i, "samples", tot_s)
k = int(sys.argv[2]) if len(sys.argv) > 2 else 40
idx = {r[0]: n for n, r in enumerate(data)}
for key, lab in ((ss, "stall"), (ia, "instr")):
    print("== top by", lab)
    for r in sorted(data, key=lambda r: -int(r[key] or 0))[:k]:
        print(f"{idx[r[0]]:5d} {int(r[ia] or 0):10d} {int(r[ss] or 0):7d}  {r[1].strip()[:90]}")
