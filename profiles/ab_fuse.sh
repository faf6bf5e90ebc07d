mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for f in 0 1; do
  WG_FUSE_INSERT=$f timeout 600 python bench.py --steps 50 --warmup 5 --cpu-sample-s 0 > gpurun_out/bench_f$f.log 2>&1; echo bench$f=$?
  python -c "import json;d=json.loads(open('gpurun_out/bench_f$f.log').read().strip().splitlines()[-1]);print('fuse',$f,d['value'],d['ms_per_step'],d['roofline']['frac'],d['roofline']['gather_ms_per_step'])"
  WG_FUSE_INSERT=$f timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_f$f.csv python bench.py --steps 2 --warmup 3 --cpu-sample-s 0 --e2e-steps 1 > /dev/null 2>&1
done
