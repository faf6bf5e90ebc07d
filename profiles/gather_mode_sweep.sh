#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for F in 0 1; do for P in 1 4 8; do
WG_GATHER_FLAT=$F timeout 600 python bench.py --steps 50 --warmup 5 --cpu-sample-s 0 --concurrency $P > gpurun_out/bench_f${F}_p$P.log 2>&1
python -c "import json;d=json.loads(open('gpurun_out/bench_f${F}_p$P.log').read().strip().splitlines()[-1]);print('flat',$F,'P',$P,round(d['value']),round(d['ms_per_step'],4),round(d['single_batch']['ms_per_batch'],4),round(d['roofline']['frac'],3),round(d['roofline']['gather_ms_per_launch'],4))"
done; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 --concurrency 1 > /dev/null 2>&1
echo done
