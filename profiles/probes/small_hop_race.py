"""Repeat one products hop-0 batch through wg_sample_hop and count runs whose unique list differs from the
oracle (race hunt for the cluster hop)."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import oracle
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import presets, seeds, providers
p = presets.get("products")
dsm, _ = loader.build_dsm(p, on_device=True)
rows = providers.host_row_provider(p.graph())
pipe = pkg.MiniBatchPipeline(dsm, p.fanouts[:1], p.seeds_per_batch, with_dup=True, incremental_gather=False)
bad = 0
N = int(sys.argv[1]) if len(sys.argv) > 1 else 40
refs = {}
for r in range(N):
    b = r % 4
    S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
    rs = seeds.rng_seed(presets.RNG_BASE, b)
    if b not in refs:
        ap, adj = rows(S)
        o_rp, o_nb, o_pos = oracle.sample_hop(ap, adj, S, p.fanouts[0], rs, 0)
        refs[b] = oracle.append_unique(S, o_nb)
    pipe.set_inputs(torch.from_numpy(S).cuda(), rs)
    pipe.enqueue(gather=False)
    torch.cuda.synchronize()
    got = pipe.result(0)
    U, sc, dup = refs[b]
    bad += not (np.array_equal(got["unique"], U) and np.array_equal(got["sub_col"], sc) and np.array_equal(got["dup"], dup))
print(os.path.basename(os.getcwd()), "bad", bad, "of", N, "err", dsm.device_error(), flush=True)
