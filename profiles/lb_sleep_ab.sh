#!/bin/bash
# A/B of the decoupled look-back back-off (WG_LB_SLEEP_NS = 0 / 32 / 128), prebuilt .so variants in abso/,
# interleaved runs so clock/thermal drift hits every variant alike; default bench config (P=8) + single batch.
mkdir -p gpurun_out
L=paper_conf_sc_yanglql22_b200/libwg.so
for r in 1 2; do for V in spin32 spin0 spin128; do
cp abso/libwg_$V.so $L
timeout 300 python bench.py --steps 50 --warmup 5 --cpu-sample-s 0 --e2e-steps 10 > gpurun_out/b.log 2>&1
echo -n "$V r$r "; python profiles/bench_summary.py gpurun_out/b.log
done; done
# restore the default build from source (never a copied binary: _build.py stamps the flags + hash)
python -c "from paper_conf_sc_yanglql22_b200 import _build; _build.build_lib(force=True)"
