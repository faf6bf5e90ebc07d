#!/bin/bash
# compact 8 B hash slots (default) vs 16 B slots (WG_HASH_COMPACT=0): GPU tests + throughput pass
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_compact.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_compact.log
WG_HASH_COMPACT=0 timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -1
for rep in 1 2 3; do for C in 1 0; do
  WG_HASH_COMPACT=$C timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/hc.log 2>&1
  echo "compact=$C $(python profiles/bench_summary.py gpurun_out/hc.log 2>&1 | tail -1)"
done; done
