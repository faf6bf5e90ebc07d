#!/bin/bash
# end-of-round check: GPU tests, smoke, default bench (N=1), oracle arm, 2-rank torchrun bench, launch list
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py > gpurun_out/bench_default.log 2>&1; echo bench=$?; python profiles/bench_summary.py gpurun_out/bench_default.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.log 2>&1; echo ref=$?; tail -c 300 gpurun_out/bench_reference.log
bash profiles/w2_same_gpu.sh
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 > /dev/null 2>&1
python profiles/launches_table.py gpurun_out/launches.csv
