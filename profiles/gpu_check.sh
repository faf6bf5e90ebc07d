#!/bin/bash
# tests + bench + launch list (one gpurun call)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 50 --warmup 5 --cpu-sample-s ${CPU_S:-0} ${BENCH_ARGS:-} > gpurun_out/bench.log 2>&1; echo bench=$?
python -c "import json;d=json.loads(open('gpurun_out/bench.log').read().strip().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['roofline']['gather_ms_per_step'])"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 ${BENCH_ARGS:-} > /dev/null 2>&1
python - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/launches.csv')))
for i,r in enumerate(rows):
    if r and r[0]=='ID': hdr=r; start=i; break
idx={k:j for j,k in enumerate(hdr)}
for r in rows[start+1:][-16:]:
    print('  ',r[idx['Kernel Name']][:60], r[idx['Metric Value']])
PY
