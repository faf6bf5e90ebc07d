#!/usr/bin/env python
"""One products-shaped batch for ncu: 3 warm-up batches, then one batch whose kernels (3 hops x
sample/flag/relabel with the direct key table, + insert with a hashed one; then the whole gather) are the
ones to capture:

    ncu --set full -k regex:'sample_kernel|unique_|gather_kernel' -s 30 -c 10 python profiles/ncu_step.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yanglql22_b200 as pkg  # noqa: E402
from paper_conf_sc_yanglql22_b200 import loader  # noqa: E402
from synth import presets, seeds  # noqa: E402

p = presets.get(sys.argv[1] if len(sys.argv) > 1 else "products")
dsm, _ = loader.build_dsm(p)
pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, incremental_gather=False)
for b in range(4):
    pipe.run(torch.from_numpy(seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)).cuda(),
             seeds.rng_seed(presets.RNG_BASE, b))
    torch.cuda.synchronize()
print("rows_gathered", int(pipe.hops[-1]["num_unique"].item()), "row_bytes", dsm.row_bytes)
dsm.destroy()
