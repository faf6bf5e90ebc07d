#!/bin/bash
# per-call hash-table prefix of factor x the call's key bound slots (WG_HASH_FACTOR), throughput pass
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for rep in 1 2; do for F in 1.25 1.5 2 3; do
  WG_HASH_FACTOR=$F timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/hpc.log 2>&1
  echo "F=$F $(python profiles/bench_summary.py gpurun_out/hpc.log)"
done; done
