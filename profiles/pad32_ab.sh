#!/bin/bash
# uint32 padded sampler slots (WG_PAD32, default 1) vs int64: GPU tests + throughput pass
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_pad32.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_pad32.log
WG_PAD32=0 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "tiny or sample or hop" 2>&1 | tail -1
for rep in 1 2 3; do for C in 1 0; do
  WG_PAD32=$C timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 3 > gpurun_out/p32.log 2>&1
  echo "pad32=$C $(python profiles/bench_summary.py gpurun_out/p32.log 2>&1 | tail -1)"
done; done
