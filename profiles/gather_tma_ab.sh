#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gather" > gpurun_out/pytest_gather.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gather.log
for T in 0 1; do for P in 1 8; do
WG_GATHER_TMA=$T timeout 600 python bench.py --steps 40 --warmup 5 --cpu-sample-s 0 --e2e-steps 2 --concurrency $P > gpurun_out/b.log 2>&1
python -c "import json;d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]);print('tma',$T,'P',$P,round(d['value']),round(d['ms_per_step'],4),round(d['single_batch']['ms_per_batch'],4),round(d['roofline']['frac'],3),round(d['roofline']['gather_ms_per_launch'],4))" || tail -5 gpurun_out/b.log
done; done
WG_GATHER_TMA=1 timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_tma.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 > /dev/null 2>&1
python profiles/launches_table.py gpurun_out/launches_tma.csv 1
