#!/bin/bash
# per-call hash-table prefix (WG_HASH_PER_CALL, WG_HASH_MIN_SLOTS) x table factor (WG_HASH_FACTOR), throughput pass
mkdir -p gpurun_out
for rep in 1 2; do for cfg in "0 2 0" "1 1.5 1024" "1 1.5 524288" "1 1.5 1048576" "1 1.5 2097152" "1 2 1048576"; do set -- $cfg
  WG_HASH_PER_CALL=$1 WG_HASH_FACTOR=$2 WG_HASH_MIN_SLOTS=$3 timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/hpc.log 2>&1
  echo "per_call=$1 F=$2 min_slots=$3 $(python profiles/bench_summary.py gpurun_out/hpc.log)"
done; done
