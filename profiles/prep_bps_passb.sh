#!/bin/bash
# insert/relabel grid cap (WG_PREP_BPS blocks per SM) in the throughput pass (gather occupancy 1)
mkdir -p gpurun_out
for rep in 1 2; do for B in 8 4 2; do
  WG_PREP_BPS=$B timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/pbps_$B.log 2>&1
  echo "prep_bps=$B $(python profiles/bench_summary.py gpurun_out/pbps_$B.log)"
done; done
