"""Run a few products batches (one batch at a time, L2 flushed) through the shipped graph of a
WG_FLAG_TIMING=1 build: the flag scan of hop 2 prints when its tiles started, published their aggregate
and finished, as 8-bin histograms over the kernel's span."""
import os, sys
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import presets, seeds
p = presets.get("products")
dsm, _ = loader.build_dsm(p)
pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for b in range(6):
    flush.fill_(b)
    pipe.run(torch.from_numpy(seeds.seed_nodes(p.n, 1024, presets.SEED_BASE, b)).cuda(), seeds.rng_seed(presets.RNG_BASE, b))
    torch.cuda.synchronize()
    if b == 1:
        pipe.capture()
