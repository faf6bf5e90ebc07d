#!/bin/bash
# TMA bulk-copy gather (bytes in flight in shared memory, one warp per block) vs the LSU gather in pass B
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "tma or gather_rows" 2>&1 | tail -2
for rep in 1 2; do for cfg in "0 0" "1 0" "1 2" "1 1"; do set -- $cfg
  WG_GATHER_TMA=$1 WG_GATHER_BPS=$2 timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/gtma_$1_$2.log 2>&1
  echo "tma=$1 bps=$2 $(python profiles/bench_summary.py gpurun_out/gtma_$1_$2.log)"
done; done
