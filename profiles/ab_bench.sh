#!/bin/bash
# Interleaved A/B of two builds: the working tree (B) and ab_old/ (A, built beforehand with other defines),
# default bench config (products, P=8), $REPS rounds; prints value (M seeds/s), gather frac, single-batch ms.
mkdir -p gpurun_out
summ() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); s=d.get('stages_ms') or {}
print('$2', round(d['value']/1e6,3), round(d['roofline']['frac'],3), round(d['single_batch']['ms_per_batch'],4), round(d['whole_step_roofline']['frac'],3), ' '.join(f'{k}={v*1e3:.1f}' for k,v in s.items() if k.startswith('hop') and '_' in k))"; }
for r in $(seq 1 ${REPS:-2}); do
  (cd ab_old && timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 5 --north-star "" --no-parity ${ARGS:-} > ../gpurun_out/ab_A_$r.log 2>&1); summ gpurun_out/ab_A_$r.log "A r$r"
  timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 5 --north-star "" --no-parity ${ARGS:-} > gpurun_out/ab_B_$r.log 2>&1; summ gpurun_out/ab_B_$r.log "B r$r"
done
