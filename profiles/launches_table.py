#!/usr/bin/env python
"""Print the last step's kernels from an ncu --csv launch list (one row per kernel)."""
import csv
import sys
from collections import OrderedDict

rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 13  # bench.py ends with its stage breakdown: one batch = (sample, insert, flag, relabel) x 3 hops + the whole gather
for i, r in enumerate(rows):
    if r and r[0] == "ID":
        hdr, start = r, i
        break
idx = {k: j for j, k in enumerate(hdr)}
kern = OrderedDict()
for r in rows[start + 1:]:
    d = kern.setdefault(r[idx["ID"]], {"name": r[idx["Kernel Name"]]})
    d[r[idx["Metric Name"]]] = (r[idx["Metric Value"]], r[idx["Metric Unit"]])
items = [v for v in kern.values() if "wg::" in v["name"]][-n:]
tot = 0.0
for v in items:
    t = float(v["gpu__time_duration.sum"][0].replace(",", ""))
    tu = v["gpu__time_duration.sum"][1]
    t_us = t / 1000 if tu == "ns" else (t if tu == "us" else t * 1000)
    tot += t_us
    extra = ""
    if "dram__bytes_read.sum" in v:
        extra = f"  read {v['dram__bytes_read.sum'][0]} {v['dram__bytes_read.sum'][1]}  write {v['dram__bytes_write.sum'][0]} {v['dram__bytes_write.sum'][1]}"
    print(f"{t_us:9.2f} us  {v['name'][:70]}{extra}")
print(f"{tot:9.2f} us total")
