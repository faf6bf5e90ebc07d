#!/bin/bash
# row_ptr loads with an L2 evict_last hint (WG_RP_EVICT_LAST) in the throughput pass
mkdir -p gpurun_out
for rep in 1 2 3; do for K in 0 1; do
  WG_RP_EVICT_LAST=$K timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/rpk.log 2>&1
  echo "rp_keep=$K $(python profiles/bench_summary.py gpurun_out/rpk.log)"
done; done
