#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
for E in 1 0; do for P in 1 8; do
WG_PDL=$E timeout 600 python bench.py --steps 50 --warmup 5 --cpu-sample-s 0 --e2e-steps 10 --concurrency $P > gpurun_out/b.log 2>&1
echo -n "pdl=$E "; python profiles/bench_summary.py gpurun_out/b.log
done; done
