#!/bin/bash
# throughput-pass gather occupancy (wg_dsm_set_gather_occupancy) sweep: pass A (roofline) unchanged
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for rep in 1 2; do for O in 0 1 2; do for P in 8 12; do
  timeout 600 python bench.py --cpu-sample-s 0 --e2e-steps 5 --gather-occupancy $O --concurrency $P > gpurun_out/gocc_$O.log 2>&1
  echo "occ=$O $(python profiles/bench_summary.py gpurun_out/gocc_$O.log)"
done; done; done
