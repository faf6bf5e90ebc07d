#!/bin/bash
mkdir -p gpurun_out
for M in 0 1 2 3 4; do for S in 0 1; do
WG_GATHER_LD=$M WG_GATHER_ST=$S timeout 600 python bench.py --steps 40 --warmup 5 --cpu-sample-s 0 --e2e-steps 2 --concurrency 1 > gpurun_out/b.log 2>&1
echo -n "ld=$M st=$S "; python profiles/bench_summary.py gpurun_out/b.log
done; done
for M in 0 4; do
WG_GATHER_LD=$M timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:gather --csv --log-file gpurun_out/launches_ld$M.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 > /dev/null 2>&1
echo "ld=$M"; python profiles/launches_table.py gpurun_out/launches_ld$M.csv 1
done
