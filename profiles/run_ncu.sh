#!/bin/bash
# Profiling recipe (run on the GPU box under gpurun; see /opt/skills/guides/B200_PROFILING.md).
# 1) launch list of one default bench invocation (every kernel, device time, serialized)
# 2) one `ncu --set full` capture of the 13 kernels of one products-shaped batch (profiles/ncu_step.py)
set -u
OUT=${1:-gpurun_out}
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 > $OUT/ncu_launches_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:'sample_kernel|unique_|gather_kernel' \
    -s 39 -c 13 -o $OUT/prof_step -f python profiles/ncu_step.py > $OUT/ncu_full_step.log 2>&1
grep rows_gathered $OUT/ncu_full_step.log
echo done
