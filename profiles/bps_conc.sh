#!/bin/bash
mkdir -p gpurun_out
for B in 0 4 3 2; do for P in 4 8; do
WG_GATHER_BPS=$B timeout 600 python bench.py --steps 40 --warmup 5 --cpu-sample-s 0 --e2e-steps 2 --concurrency $P > gpurun_out/b.log 2>&1
echo -n "bps=$B "; python profiles/bench_summary.py gpurun_out/b.log
done; done
