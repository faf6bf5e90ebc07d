"""Seeded randomized parity campaign (tolerance 0 against the oracle): random graphs (power-law degrees with
planted hubs, empty rows, self-loop-free sorted rows), random fan-out lists (1-4 hops, 1..40 per hop: both
samplers), random seed counts (0, 1, ragged), every layout / placement flag, W in {1, 2, 3} virtual ranks,
eager runs and CUDA-graph replays, with and without positions / duplicate counts."""

import threading

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200.pipeline import required_keys
from synth import features, presets, providers

from gpu_helpers import csr_from_rows

pytestmark = pytest.mark.gpu

FLAG_SETS = [0, pkg.WG_DSM_COL32, pkg.WG_DSM_WIDE_HASH, pkg.WG_DSM_PAD64 | pkg.WG_DSM_COL32,
             pkg.WG_DSM_WHOLE_ROWS, pkg.WG_DSM_CSR_REPLICATED | pkg.WG_DSM_COL32, pkg.WG_DSM_CSR_REPLICATED,
             pkg.WG_DSM_HASHED | pkg.WG_DSM_COL32, pkg.WG_DSM_HASHED | pkg.WG_DSM_PAD64]


def _random_graph(rng, n):
    deg = np.minimum((rng.pareto(1.3, n) * rng.uniform(1, 6)).astype(np.int64), n - 1)
    deg[rng.choice(n, max(1, n // 50), replace=False)] = 0                  # empty rows
    hubs = rng.choice(n, 3, replace=False)
    rows = []
    for v in range(n):
        d = int(deg[v])
        if d == 0:
            rows.append(np.zeros(0, np.int64))
            continue
        # destinations skewed toward the planted hubs (repeated ids across rows)
        cand = np.concatenate([rng.integers(0, n, d), rng.choice(hubs, max(1, d // 3))])
        r = np.unique(cand)
        rows.append(r[r != v][: n - 1])
    return csr_from_rows(rows)


def _make(rp, col, n, dim, dtype, flags, W, max_keys):
    feat = features.feature_bytes(presets.FEAT_SEED, np.arange(n), dim, dtype)
    ag = pkg.ThreadAllgather(W) if W > 1 else None
    out, errs = [None] * W, []

    def create(r):
        try:
            rep = bool(flags & pkg.WG_DSM_CSR_REPLICATED)
            e_local = len(col) if rep else pkg.local_num_edges(rp, r, W)
            d = pkg.DSM(n, e_local, dim, dtype, max_keys, rank=r, world_size=W,
                        allgather=ag.for_rank(r) if ag else None, flags=flags)
            d.fill_from_global_csr(rp, col)
            d.fill_features(feat[r::W])
            torch.cuda.synchronize()
            if ag:
                ag.for_rank(r)(None, None, 0, None)
            out[r] = d
        except Exception as e:  # pragma: no cover
            errs.append(e)
    ths = [threading.Thread(target=create, args=(r,)) for r in range(W)]
    [t.start() for t in ths]
    [t.join() for t in ths]
    assert not errs, errs
    return out, feat


@pytest.mark.parametrize("case", range(96))
def test_random_pipelines_bit_exact(case):
    rng = np.random.default_rng(1000 + case)
    n = int(rng.integers(50, 3000))
    rp, col = _random_graph(rng, n)
    H = int(rng.integers(1, 5))
    fan = [int(rng.choice([1, 2, 3, 5, 8, 9, 15, 16, 17, 25, 32, 33, 40])) for _ in range(H)]
    max_seeds = int(rng.integers(1, min(n, 200) + 1))
    dim, dtype = [(8, "fp32"), (100, "fp32"), (36, "fp16"), (3, "fp32"), (64, "bf16")][case % 5]
    flags = FLAG_SETS[case % len(FLAG_SETS)]
    W = [1, 2, 3][case % 3]
    with_pos, with_dup = bool(case & 1), bool(case & 2)
    keys = required_keys(n, fan, max_seeds)
    dsms, feat = _make(rp, col, n, dim, dtype, flags, W, keys)
    rows = providers.host_row_provider(None, rp, col)

    def feats(ids):
        u = np.unique(np.asarray(ids, dtype=np.int64))
        return u, feat[u]
    try:
        for r, dsm in enumerate(dsms):
            pipe = pkg.MiniBatchPipeline(dsm, fan, max_seeds, with_pos=with_pos, with_dup=with_dup)
            for b in range(3):
                cnt = [max_seeds, 0, 1][b] if case % 4 == 0 else int(rng.integers(0, max_seeds + 1))
                S = rng.choice(n, cnt, replace=False).astype(np.int64)
                rs = int(rng.integers(0, 2 ** 63))
                pipe.run(torch.from_numpy(S).cuda() if cnt else torch.zeros(0, dtype=torch.int64, device="cuda"), rs)
                torch.cuda.synchronize()
                ref = oracle.minibatch(rows, feats, S, fan, rs)
                for h in range(H):
                    got, exp = pipe.result(h), ref["hops"][h]
                    keys_ = ["row_ptr", "nbrs", "unique", "sub_col"] + (["pos"] if with_pos else []) + \
                        (["dup"] if with_dup else [])
                    for k in keys_:
                        assert np.array_equal(got[k], exp[k]), (case, r, b, h, k, fan, flags, W)
                assert np.array_equal(pipe.features(), ref["X"]), (case, r, b)
                if b == 0 and max(fan) <= 32:
                    pipe.capture()          # later batches replay the captured graph
            assert dsm.device_error() == 0, (case, r)
            del pipe
    finally:
        if len(dsms) > 1:
            ths = [threading.Thread(target=d.destroy) for d in dsms]
            [t.start() for t in ths]
            [t.join() for t in ths]
        else:
            dsms[0].destroy()


@pytest.mark.parametrize("case", range(32))
def test_random_standalone_ops_bit_exact(case):
    """wg_sample_neighbors then wg_append_unique (the separate ops, dense layouts) and wg_gather on random
    graphs, fan-outs and target lists: every output against the oracle."""
    rng = np.random.default_rng(5000 + case)
    n = int(rng.integers(20, 2000))
    rp, col = _random_graph(rng, n)
    M = int(rng.choice([1, 4, 5, 10, 16, 31, 32, 33, 64, 129]))
    nT = int(rng.integers(0, min(n, 300) + 1))
    T = rng.choice(n, nT, replace=False).astype(np.int64)
    flags = [0, pkg.WG_DSM_COL32, pkg.WG_DSM_WIDE_HASH, pkg.WG_DSM_PAD64, pkg.WG_DSM_HASHED][case % 5]
    dsms, feat = _make(rp, col, n, 12, "fp32", flags, 1, max(nT * (M + 1), 1))
    dsm = dsms[0]
    try:
        seed, hop = int(rng.integers(0, 2 ** 63)), int(rng.integers(0, 4))
        t = torch.from_numpy(T).cuda() if nT else torch.zeros(0, dtype=torch.int64, device="cuda")
        rpo, nb, pos, ne = dsm.sample_neighbors(t, M, seed, hop, with_pos=True)
        torch.cuda.synchronize()
        e = int(ne.item())
        adj_ptr, adj = providers.host_row_provider(None, rp, col)(T)
        o_rp, o_nb, o_pos = oracle.sample_hop(adj_ptr, adj, T, M, seed, hop)
        assert np.array_equal(rpo[: nT + 1].cpu().numpy(), o_rp) and np.array_equal(nb[:e].cpu().numpy(), o_nb)
        assert np.array_equal(pos[:e].cpu().numpy(), o_pos)
        U, nU, sc, dup = dsm.append_unique(t, nb[:max(e, 1)] if e else torch.zeros(0, dtype=torch.int64, device="cuda"),
                                           n_nbrs=e, with_dup=True)
        torch.cuda.synchronize()
        u = int(nU.item())
        Uo, sco, dupo = oracle.append_unique(T, o_nb)
        assert np.array_equal(U[:u].cpu().numpy(), Uo) and np.array_equal(sc[:e].cpu().numpy(), sco)
        assert np.array_equal(dup[:u].cpu().numpy(), dupo)
        if u:
            X = dsm.gather(U[:u])
            torch.cuda.synchronize()
            assert np.array_equal(X[:u].cpu().numpy(), feat[Uo])
        assert dsm.device_error() == 0
    finally:
        dsm.destroy()
