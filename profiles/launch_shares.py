#!/usr/bin/env python
"""Aggregate an ncu --csv launch list (gpu__time_duration per launch) by kernel: launches, total and mean
device time, share of this library's kernel time.  The launch list is serialized and cold-cache, so the
SHARES (not the absolute times) compare with bench.py's CUDA-event timing."""
import csv
import re
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
hdr = rows[0]
idx = {k: j for j, k in enumerate(hdr)}
agg = defaultdict(lambda: [0, 0.0])
for r in rows[1:]:
    if r[idx["Metric Name"]] != "gpu__time_duration.sum" or "wg::" not in r[idx["Kernel Name"]]:
        continue
    t = float(r[idx["Metric Value"]].replace(",", ""))
    u = r[idx["Metric Unit"]]
    t_us = t / 1000 if u in ("ns", "nsecond") else (t if u in ("us", "usecond") else t * 1000)
    name = re.sub(r"\(.*", "", r[idx["Kernel Name"]]).replace("void ", "")
    agg[name][0] += 1
    agg[name][1] += t_us
tot = sum(v[1] for v in agg.values())
print(f"{sys.argv[1]}: {sum(v[0] for v in agg.values())} wg:: launches, {tot:.0f} us of device time\n")
print("| kernel | launches | total us | mean us | share |")
print("|---|---|---|---|---|")
for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"| `{k}` | {n} | {t:.0f} | {t / n:.2f} | {t / tot:.3f} |")
