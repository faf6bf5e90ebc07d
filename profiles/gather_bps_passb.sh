#!/bin/bash
# Does leaving SM room next to the gather let other streams' prep kernels overlap it?
# WG_GATHER_BPS = gather blocks per SM (default: occupancy max, 4 x 256 threads at 60 regs)
mkdir -p gpurun_out
for rep in 1 2; do for B in 4 3 2 1; do
  WG_GATHER_BPS=$B timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/gbps_$B.log 2>&1
  echo "bps=$B $(python profiles/bench_summary.py gpurun_out/gbps_$B.log)"
done; done
