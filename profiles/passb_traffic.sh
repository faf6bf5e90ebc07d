#!/bin/bash
# DRAM bytes and time of the concurrent throughput pass as one graph (profiles/ncu_passb.py)
mkdir -p gpurun_out
for m in ${MODES:-both prep gather}; do
  for P in ${PS:-8}; do
    timeout 300 python profiles/ncu_passb.py $m $P 2>&1 | grep mode=
    REPS=2 timeout 300 ncu --graph-profiling graph --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_op_read.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum \
      --clock-control none --csv --log-file gpurun_out/passb_${m}_$P.csv python profiles/ncu_passb.py $m $P > /dev/null 2>&1
    python - gpurun_out/passb_${m}_$P.csv $m $P <<'PY'
import csv, sys
lines = [l for l in open(sys.argv[1]) if l.startswith('"')]
rows = list(csv.DictReader(lines))
ids = sorted({r["ID"] for r in rows}, key=int)
last = ids[-1]
m = {r["Metric Name"]: (r["Metric Unit"], float(r["Metric Value"].replace(",", ""))) for r in rows if r["ID"] == last}
mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "usecond": 1e-6, "msecond": 1e-3, "nsecond": 1e-9}
def v(k):
    u, x = m[k]
    return x * mult.get(u, 1)
P = int(sys.argv[3])
rd, wr, t = v("dram__bytes_read.sum"), v("dram__bytes_write.sum"), v("gpu__time_duration.sum")
print(f"ncu graph {sys.argv[2]} P={P}: {t*1e6:.1f} us, DRAM read {rd/P/1e6:.1f} MB + write {wr/P/1e6:.1f} MB per batch, "
      f"{(rd+wr)/t/1e9:.0f} GB/s; L2 sectors read {m['lts__t_sectors_op_read.sum'][1]/P/1e6:.2f}M atom {m['lts__t_sectors_op_atom.sum'][1]/P/1e6:.2f}M red {m['lts__t_sectors_op_red.sum'][1]/P/1e6:.2f}M per batch")
PY
  done
done
