#!/bin/bash
# A/B of the sampler block size (WG_SAMPLE_THREADS = 128 / 256 / 512, SAMPLE_MINB keeping the register cap), prebuilt .so variants in abso/:
# parity subset per variant, then interleaved default-config bench runs.
mkdir -p gpurun_out
L=paper_conf_sc_yanglql22_b200/libwg.so
for V in st128 st512; do
cp abso/libwg_$V.so $L
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "sample or tiny_pipeline or degenerate" 2>&1 | tail -1 | sed "s/^/$V parity: /"
done
for r in 1 2; do for V in st256 st128 st512; do
cp abso/libwg_$V.so $L
timeout 300 python bench.py --steps 50 --warmup 5 --cpu-sample-s 0 --e2e-steps 10 > gpurun_out/b.log 2>&1
echo -n "$V r$r "; python profiles/bench_summary.py gpurun_out/b.log
done; done
# restore the default build from source (never a copied binary: _build.py stamps the flags + hash)
python -c "from paper_conf_sc_yanglql22_b200 import _build; _build.build_lib(force=True)"
