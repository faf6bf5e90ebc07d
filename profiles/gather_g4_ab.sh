#!/bin/bash
# TMA gather4 gather (WG_GATHER_G4=1) vs the LSU gather: parity, pass A roofline, pass B throughput
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "tma_variant" 2>&1 | tail -2
for rep in 1 2; do for cfg in "0 1" "1 0" "1 1"; do set -- $cfg
  WG_GATHER_G4=$1 timeout 300 python bench.py --cpu-sample-s 0 --e2e-steps 3 --gather-occupancy $2 > gpurun_out/g4.log 2>&1
  echo "g4=$1 occ=$2 $(python profiles/bench_summary.py gpurun_out/g4.log 2>&1 | tail -1)"
done; done
