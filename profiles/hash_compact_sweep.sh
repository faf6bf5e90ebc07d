#!/bin/bash
# compact table: factor x min-slots sweep, throughput pass (products), then papers100M at the default
mkdir -p gpurun_out
for rep in 1 2; do for cfg in "2 1048576" "3 1048576" "4 1048576" "1.5 1048576" "2 262144" "3 262144"; do set -- $cfg
  WG_HASH_FACTOR=$1 WG_HASH_MIN_SLOTS=$2 timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/hcs.log 2>&1
  echo "F=$1 min=$2 $(python profiles/bench_summary.py gpurun_out/hcs.log 2>&1 | tail -1)"
done; done
