mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for P in 1 2 3 4 6; do
timeout 600 python bench.py --steps 50 --warmup 5 --cpu-sample-s 0 --concurrency $P > gpurun_out/bench_p$P.log 2>&1; echo bench=$?
python -c "import json;d=json.loads(open('gpurun_out/bench_p$P.log').read().strip().splitlines()[-1]);print('P',$P,d['value'],d['ms_per_step'],d['single_batch'],d['roofline']['frac'])"
done
