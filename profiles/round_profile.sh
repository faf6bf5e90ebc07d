#!/bin/bash
# Round-end profiling of the shipped build (run on the GPU box under gpurun):
# 1) the ncu launch list of the bench command itself (the driver's shape, --steps 2 --warmup 1;
#    serialized, cold: shares, not absolute times, are comparable with the bench's timing)
# 2) ncu --set full of one batch's 13 kernels for products and papers100M (profiles/run_ncu.sh)
mkdir -p gpurun_out
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches_bench.csv \
    python bench.py --steps 2 --warmup 1 > gpurun_out/ncu_launches_bench.log 2>&1; echo launches=$?
for C in products papers100m; do SKIP_LAUNCHES=1 CONFIG=$C timeout 1200 bash profiles/run_ncu.sh gpurun_out; done
