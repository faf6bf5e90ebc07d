#!/bin/bash
# tests + bench (concurrency 1/4/8) + launch list, in one gpurun call
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for P in ${PS:-1 4 8}; do
  timeout 600 python bench.py --steps 50 --warmup 5 --cpu-sample-s ${CPU_S:-0} --concurrency $P ${BENCH_ARGS:-} > gpurun_out/bench_p$P.log 2>&1; echo bench=$?
  python profiles/bench_summary.py gpurun_out/bench_p$P.log
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 ${BENCH_ARGS:-} > /dev/null 2>&1
python profiles/launches_table.py gpurun_out/launches.csv
