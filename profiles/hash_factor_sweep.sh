#!/bin/bash
mkdir -p gpurun_out
for F in 1.5 2 3 4; do for P in 1 8; do
WG_HASH_FACTOR=$F timeout 600 python bench.py --steps 40 --warmup 5 --cpu-sample-s 0 --e2e-steps 2 --concurrency $P > gpurun_out/b.log 2>&1
echo -n "factor=$F "; python profiles/bench_summary.py gpurun_out/b.log
done; done
