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
pipe = pkg.MiniBatchPipeline(dsm, p.fanouts[:1], p.seeds_per_batch, with_pos=True, with_dup=True, incremental_gather=False)
for b in [1, 0, 1, 2]:
    S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
    rs = seeds.rng_seed(presets.RNG_BASE, b)
    pipe.set_inputs(torch.from_numpy(S).cuda(), rs)
    pipe.enqueue(gather=False)
    torch.cuda.synchronize()
    got = pipe.result(0)
    ap, adj = rows(S)
    o_rp, o_nb, o_pos = oracle.sample_hop(ap, adj, S, p.fanouts[0], rs, 0)
    U, sc, dup = oracle.append_unique(S, o_nb)
    ok = {k: np.array_equal(got[k], e) for k, e in (("row_ptr", o_rp), ("nbrs", o_nb), ("unique", U), ("sub_col", sc), ("dup", dup))}
    msg = ""
    if not ok["unique"]:
        g = got["unique"]
        d = np.nonzero(g[:len(U)] != U[:len(g)])[0]
        msg = f"len {len(g)} vs {len(U)} first_diff {d[:5]} nT {len(S)} sets_equal {set(g.tolist()) == set(U.tolist())}"
        i = d[0]
        msg += f" got {g[i-2:i+3]} exp {U[i-2:i+3]}"
        x = U[i]
        occ = np.nonzero(o_nb == x)[0]
        msg += f"\n   key {x}: occurrences {occ[:8]} (nT+pos) ; got sub_col {got['sub_col'][occ[:8]]} exp {sc[occ[:8]]}; got index of key {np.nonzero(g == x)[0]}"
        # padded position of the first occurrence: target k = row of occ[0]
        k = np.searchsorted(o_rp, occ[0], side='right') - 1
        msg += f"; first occ target k={k} deg-slot {occ[0]-o_rp[k]} cnt {o_rp[k+1]-o_rp[k]}"
    print(b, ok, msg, "err", dsm.device_error(), flush=True)
