#!/bin/bash
# Profiling recipe (run on the GPU box under gpurun; see /opt/skills/guides/B200_PROFILING.md).
# 1) launch list of one bench invocation: every kernel with its device time
# 2) one `ncu --set full` capture of each hot kernel of one timed step
set -u
OUT=${1:-gpurun_out}
mkdir -p $OUT
BENCH="python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 ${BENCH_ARGS:-}"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv $BENCH > $OUT/ncu_launches_bench.log 2>&1
# skip the eager warm-up + graph warm-up launches (13 per step x 6) and profile one timed step
ncu --set full --clock-control none --import-source on -k regex:'sample_kernel|unique_|gather_kernel' \
    -s 78 -c 13 -o $OUT/prof_step -f $BENCH > $OUT/ncu_full_bench.log 2>&1
echo done
