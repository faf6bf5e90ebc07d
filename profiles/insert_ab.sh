#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
WG_INSERT_WARP=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tiny or unique" > gpurun_out/pytest_gpu_warp.log 2>&1; echo pytest_warp=$?; tail -1 gpurun_out/pytest_gpu_warp.log
for W in 0 1; do for P in 1 8; do
WG_INSERT_WARP=$W timeout 600 python bench.py --steps 50 --warmup 5 --cpu-sample-s 0 --e2e-steps 2 --concurrency $P > gpurun_out/b.log 2>&1
echo -n "warp_insert=$W "; python profiles/bench_summary.py gpurun_out/b.log
done; done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 > /dev/null 2>&1
python profiles/launches_table.py gpurun_out/launches.csv
