#!/bin/bash
# A/B of L2 persistence for the split layout's tail region (WG_TAIL_PERSIST=0/1/2, dsm.cu)
mkdir -p gpurun_out
for rep in 1 2; do
for M in 0 1 2; do
  WG_VERBOSE=1 WG_TAIL_PERSIST=$M timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 5 > gpurun_out/tp_$M.log 2>&1
  echo "persist=$M rep=$rep $(grep '\[wg\] tail' gpurun_out/tp_$M.log | head -1)"
  python profiles/bench_summary.py gpurun_out/tp_$M.log
done
done
