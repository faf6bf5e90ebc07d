"""Summarise fetch_probe ncu csv files: DRAM bytes read per gathered row, per cell (3rd launch)."""
import csv
import sys
from collections import defaultdict

CELLS = [32, 64, 96, 128, 256, 384, 400, 400, 416, 448, 512]
R = 1_000_000
for path in sys.argv[1:]:
    rows = defaultdict(dict)
    order = []
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    for r in csv.DictReader(lines):
        k = r["ID"]
        if k not in rows:
            order.append(k)
        v = r["Metric Value"].replace(",", "")
        rows[k][r["Metric Name"]] = (float(v), r["Metric Unit"])
    print(path)
    print("| row B | launch | us | dram rd B/row | dram wr B/row | L2 rd sectors/row | L2 miss sectors/row |")
    print("|---|---|---|---|---|---|---|")
    for i, k in enumerate(order):
        if i % 3 != 2:
            continue
        c = CELLS[i // 3] if i // 3 < len(CELLS) else "?"
        m = rows[k]

        def val(name, scale=1.0):
            if name not in m:
                return float("nan")
            x, u = m[name]
            mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "nsecond": 1e-3, "us": 1, "usecond": 1, "msecond": 1e3}.get(u, 1)
            return x * mult * scale
        label = f"{c}" + (" (416 B pitched out)" if i // 3 == 7 else "")
        print(f"| {label} | {k} | {val('gpu__time_duration.sum'):.1f} | {val('dram__bytes_read.sum') / R:.1f} | "
              f"{val('dram__bytes_write.sum') / R:.1f} | {val('lts__t_sectors_srcunit_tex_op_read.sum') / R:.2f} | "
              f"{val('lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum') / R:.2f} |")
