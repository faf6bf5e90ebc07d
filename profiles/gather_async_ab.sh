#!/bin/bash
# cp.async gather (bytes in flight in shared memory) vs the LSU gather: pass A roofline and pass B
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "tma_variant or occupancy" 2>&1 | tail -2
for rep in 1 2; do for cfg in "0 1" "1 0" "1 1" "1 2"; do set -- $cfg
  WG_GATHER_ASYNC=$1 timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 --gather-occupancy $2 > gpurun_out/gasync_$1_$2.log 2>&1
  echo "async=$1 occ=$2 $(python profiles/bench_summary.py gpurun_out/gasync_$1_$2.log)"
done; done
