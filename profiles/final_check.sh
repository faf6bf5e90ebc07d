#!/bin/bash
# End-of-round check: GPU tests, smoke, default bench (N=1, with the papers100M leg), oracle arm,
# 2-rank torchrun bench on the one GPU (both processes share it: gloo plumbing, parity per rank), sanitizers.
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1; echo bench=$?; python profiles/bench_summary.py gpurun_out/bench_default.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.log 2>&1; echo ref=$?; tail -c 300 gpurun_out/bench_reference.log
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29911 \
    bench.py --gpus 2 --steps 5 --warmup 3 --cpu-sample-s 0 --north-star "" > gpurun_out/bench_w2.log 2>&1; echo w2=$?
python profiles/bench_summary.py gpurun_out/bench_w2.log
# compute-sanitizer is closed on the GPU pool now (runs left GPUs needing a reset); logs from round 2 in profiles/r02/
[ "${WG_RUN_SANITIZER:-0}" = 1 ] && bash profiles/sanitize.sh
