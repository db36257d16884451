"""Fold ncu per-launch DRAM bytes into profiles/ncu_traffic.json.

usage: python tools/traffic_from_ncu.py Q14@100.0=gpurun_out/traffic/Q14_sf100.csv ...
Takes the LAST profiled launch in each CSV (the timed step's probe kernel, see
tools/ncu_traffic_sf100.sh) and stores read + write bytes under its key.
"""
import csv
import io
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def last_launch(path):
    text = open(path).read()
    start = text.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(text[start:])))
    by_id = {}
    for r in rows:
        by_id.setdefault(int(r["ID"]), {})[r["Metric Name"]] = (r["Metric Unit"], float(r["Metric Value"].replace(",", "")))
    lid = max(by_id)
    m = by_id[lid]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1024, "MB": 1024**2, "GB": 1024**3}
    tb = sum(m[k][1] * scale[m[k][0]] for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
    return lid, tb, m.get("gpu__time_duration.sum")


def main():
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    tab = json.load(open(p))
    for arg in sys.argv[1:]:
        key, path = arg.split("=", 1)
        lid, tb, dur = last_launch(path)
        tab[key] = tb
        print(key, "launch", lid, "traffic", tb, "duration", dur)
    json.dump(tab, open(p, "w"), indent=1)


if __name__ == "__main__":
    main()
