#!/bin/bash
# bench.py under torchrun with 2 ranks sharing the one GPU (setup collectives over gloo): both placements
mkdir -p gpurun_out
for PL in dsm replicas; do
  timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus 2 --steps 10 --warmup 3 --cpu-sample-s 0 --e2e-steps 2 --concurrency 4 --placement $PL > gpurun_out/w2_$PL.log 2>&1
  echo "$PL rc=$?"
  grep "^{" gpurun_out/w2_$PL.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['n_gpus'], d['config']['parallelism'], d['roofline']['bound'], round(d['roofline']['frac'],3), d['e2e']['value'], d['single_batch']['value'])"
done
