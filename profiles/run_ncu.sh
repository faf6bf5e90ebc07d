#!/bin/bash
# Profiling recipe (run on the GPU box under gpurun; see /opt/skills/guides/B200_PROFILING.md).
# 1) launch list of one default bench invocation (every kernel, device time, serialized)
# 2) one `ncu --set full` capture of the 10 (direct key table) or 13 (hashed) kernels of one batch of $CONFIG (profiles/ncu_step.py), plus the
#    L2 atomic counters SURVEY.md 8(d) names (the full set carries the sector / request counters)
set -u
OUT=${1:-gpurun_out}
CONFIG=${CONFIG:-products}
# kernels per batch: 3 hops x (sample, flag, relabel) + the gather with the direct key table (products),
# 3 hops x (sample, insert, flag, relabel) + the gather with a hashed one (papers100M: n > 2^24)
KPB=${KPB:-$([ "$CONFIG" = products ] && echo 10 || echo 13)}
mkdir -p $OUT
if [ "${SKIP_LAUNCHES:-0}" = 0 ]; then
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 --north-star "" --no-parity \
    > $OUT/ncu_launches_bench.log 2>&1
fi
ncu --set full --clock-control none --import-source on \
    --metrics lts__t_requests_op_atom_dot_cas.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum \
    -k regex:'sample_kernel|unique_|gather_kernel|gather_dense_kernel' \
    -s $((3 * KPB)) -c $KPB -o $OUT/prof_step_$CONFIG -f python profiles/ncu_step.py $CONFIG > $OUT/ncu_full_step_$CONFIG.log 2>&1
grep rows_gathered $OUT/ncu_full_step_$CONFIG.log
echo done
