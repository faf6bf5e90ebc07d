import sys, os, statistics
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import presets, seeds
p = presets.get("products")
dsm, _ = loader.build_dsm(p)
pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch)
st = torch.cuda.current_stream()
res = {}
for b in range(12):
    pipe.set_inputs(torch.from_numpy(seeds.seed_nodes(p.n, 1024, presets.SEED_BASE, b)).cuda(), seeds.rng_seed(presets.RNG_BASE, b))
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(3)]
    for row in evs:
        for e in row: e.record(st)
    tgt, tcap, tn = pipe.seeds, pipe.max_seeds, pipe.n_seeds
    for h, m in enumerate(pipe.fanouts):
        bb = pipe.hops[h]
        evs[h][0].record(st)
        dsm.set_stage_events(evs[h][1:])
        dsm.sample_hop(tgt, m, 0, h, n_targets_dev=tn, seed_dev=pipe.rng_seed, out=bb, cap=tcap, stream=st)
        dsm.set_stage_events([])
        tgt, tcap, tn = bb["unique"], pipe.U_cap[h], bb["num_unique"]
    torch.cuda.synchronize()
    if b >= 2:
        for h in range(3):
            for k, nm in enumerate(("sample", "insert", "flag", "relabel")):
                res.setdefault(f"hop{h}_{nm}", []).append(evs[h][k].elapsed_time(evs[h][k + 1]) * 1e3)
print(sys.argv[1], " ".join(f"{k}={statistics.median(v):.1f}" for k, v in res.items()))
