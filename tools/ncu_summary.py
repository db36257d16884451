"""Summarise an ncu --set full capture of the fused kernel for profiles/ (run here, no GPU)."""
import csv
import json
import subprocess
import sys


def raw(rep, which=0):
    """Metrics of the `which`-th kernel captured in the report."""
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1, "msecond": 1e3,
             "second": 1e6}
    d = {}
    for name, unit, val in zip(rows[0], rows[1], rows[2 + which]):
        if unit in scale:
            try:
                val = str(float(val.replace(",", "")) * scale[unit])  # bytes / microseconds
            except ValueError:
                pass
        d[name] = val
    return d


def sass_counts(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr = rows[1]
    src = hdr.index("Source")
    ops = {}
    for r in rows[2:]:
        op = r[src].strip().split()
        if not op:
            continue
        m = op[1] if op[0].startswith("@") and len(op) > 1 else op[0]
        m = m.split(".")[0]
        ops[m] = ops.get(m, 0) + 1
    return ops


def summarise(rep, key, which=0):
    d = raw(rep, which)
    f = lambda k: float(d[k].replace(",", "")) if k in d and d[k] not in ("", "n/a") else None
    s = {
        "workload": key,
        "kernel": d.get("Kernel Name"),
        "duration_us": f("gpu__time_duration.sum"),
        "dram_bytes_read": f("dram__bytes_read.sum"),
        "dram_bytes_write": f("dram__bytes_write.sum"),
        "dram_throughput_pct_of_peak": f("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
        "registers_per_thread": f("launch__registers_per_thread"),
        "dynamic_smem_bytes": f("launch__shared_mem_per_block_dynamic"),
        "warps_active_pct": f("sm__warps_active.avg.pct_of_peak_sustained_active"),
        "issue_active_pct": f("smsp__issue_active.avg.pct_of_peak_sustained_active"),
        "warp_instructions": f("smsp__inst_executed.sum"),
        "stall_samples": {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): int(f(k))
                          for k in d if k.startswith("smsp__pcsamp_warps_issue_stalled_") and "not_issued" not in k
                          and f(k) and f(k) > 0},
    }
    ops = sass_counts(rep) if which == 0 else {}
    s["sass_evidence"] = {k: ops.get(k, 0) for k in ("UBLKCP", "SYNCS", "LDS", "STS", "LDG", "ATOMS", "RED", "ATOMG")}
    s["traffic_bytes"] = (s["dram_bytes_read"] or 0) + (s["dram_bytes_write"] or 0)
    return s


if __name__ == "__main__":
    out = sys.argv[1]
    pairs = sys.argv[2:]  # REP KEY [REP KEY ...]; KEY may end in "#n" for the n-th kernel of REP
    res = []
    for i in range(0, len(pairs), 2):
        key = pairs[i + 1]
        which = int(key.split("#")[1]) if "#" in key else 0
        res.append(summarise(pairs[i], key, which))
    json.dump(res, open(out, "w"), indent=1)
    for r in res:
        print(json.dumps({k: r[k] for k in ("workload", "duration_us", "dram_bytes_read", "dram_bytes_write", "traffic_bytes")}))
