"""Parity of the pipelined public API (MiniBatchLoader: several batches in flight on DSM
workspace forks, graph replay, pinned-host seeds) with the CPU oracle, batch by batch."""

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import providers
from synth import graph, presets, seeds

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("depth,nb", [(1, 3), (3, 10), (4, 4)])
def test_loader_batches_bit_exact(depth, nb):
    p = presets.get("tiny")
    rp, col = graph.csr(p.graph())
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    dsm, _ = loader.build_dsm(p, on_device=False)
    ld = pkg.MiniBatchLoader(dsm, p.fanouts, p.seeds_per_batch, depth=depth, with_pos=True, with_dup=True)
    S = [seeds.seed_nodes(p.n, p.seeds_per_batch - (b % 3) * 17, presets.SEED_BASE, b) for b in range(nb)]
    rs = [seeds.rng_seed(presets.RNG_BASE, b) for b in range(nb)]
    batches = [(torch.from_numpy(s).pin_memory(), r) for s, r in zip(S, rs)]
    seen = 0
    for pb in ld(batches):
        assert pb.index == seen
        ref = oracle.minibatch(rows, feats, S[seen], p.fanouts, rs[seen])
        for h in range(len(p.fanouts)):
            got, exp = pb.hop(h), ref["hops"][h]
            for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                assert np.array_equal(got[k].cpu().numpy(), exp[k]), f"batch {seen} hop {h}: {k}"
            assert pb.counts[h] == (len(exp["nbrs"]), len(exp["unique"]))
        assert np.array_equal(pb.X.cpu().numpy(), ref["X"]), f"batch {seen}: X"
        seen += 1
    assert seen == nb
    assert ld.device_error() == 0
    ld.close()
    dsm.destroy()
