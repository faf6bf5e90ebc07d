#!/bin/bash
# hash-table factor x batches-in-flight sweep on the default products bench (pass B value)
mkdir -p gpurun_out
for F in 1.25 2; do for P in 6 8 12; do
  WG_HASH_FACTOR=$F timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 --concurrency $P > gpurun_out/hf_$F_$P.log 2>&1
  echo "F=$F $(python profiles/bench_summary.py gpurun_out/hf_$F_$P.log)"
done; done
