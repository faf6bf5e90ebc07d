#!/bin/bash
mkdir -p gpurun_out
for M in both prep gather; do for P in 1 4 8; do
timeout 600 python bench.py --steps 40 --warmup 5 --cpu-sample-s 0 --e2e-steps 2 --concurrency $P --pass-b $M > gpurun_out/b.log 2>&1
echo -n "passB=$M "; python profiles/bench_summary.py gpurun_out/b.log
done; done
