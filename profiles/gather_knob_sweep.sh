#!/bin/bash
mkdir -p gpurun_out
for U in 4 8; do for B in 0 4 3 2; do for P in 1 8; do
WG_GATHER_UNROLL=$U WG_GATHER_BPS=$B timeout 600 python bench.py --steps 40 --warmup 5 --cpu-sample-s 0 --e2e-steps 2 --concurrency $P > gpurun_out/b.log 2>&1
python -c "import json;d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]);print('unroll',$U,'bps',$B,'P',$P,round(d['value']),round(d['ms_per_step'],4),round(d['single_batch']['ms_per_batch'],4),round(d['roofline']['frac'],3),round(d['roofline']['gather_ms_per_launch'],4))"
done; done; done
