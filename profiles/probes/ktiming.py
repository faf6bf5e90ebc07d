"""Run a few products batches (one batch at a time, L2 flushed) through the shipped graph of a
WG_KTIMING=1 build (profiles/mk_ab.sh kt "-DWG_KTIMING=1"): every large launch of the sampler, insert,
flag scan and gather prints when its blocks started and ended (10-bin histograms over its span)."""
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
