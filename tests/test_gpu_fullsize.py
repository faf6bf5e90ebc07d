"""Full-size parity: the products-shaped graph (2.45M nodes, ~124M CSR entries)
generated on the device, batches of 1024 seeds through [15,10,5] + gather in the
launch configuration bench.py times (captured CUDA graphs), compared element by
element with the oracle on the same seeded inputs.  Also checks that the device
generator reproduces the host generator's rows (the inputs both sides use)."""

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import providers
from synth import features, graph, presets, seeds

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def products():
    p = presets.get("products")
    dsm, info = loader.build_dsm(p, on_device=True)
    yield p, dsm, info
    dsm.destroy()


def test_device_generator_matches_host_rows(products):
    p, dsm, info = products
    rp, col, feat = dsm.local_view()
    rng = np.random.default_rng(0)
    v = np.concatenate([[0, 1, 2, p.n - 1], rng.integers(0, p.n, 2000)]).astype(np.int64)
    hp, hc = graph.rows_native(p.graph(), v)
    rp_h = rp.cpu().numpy()
    col_d = col
    for k, x in enumerate(v):
        a, b = int(rp_h[x]), int(rp_h[x + 1])
        assert np.array_equal(col_d[a:b].cpu().numpy(), hc[hp[k]:hp[k + 1]]), x
    assert abs(rp_h[-1] - p.target_e) / p.target_e < 0.03
    fb = dsm.read_local_rows(torch.from_numpy(v).cuda()).cpu().numpy()
    assert np.array_equal(fb, features.feature_bytes(presets.FEAT_SEED, v, p.feat_dim, p.feat_dtype))


def test_products_batches_bit_exact(products):
    p, dsm, _ = products
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
    S0 = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 0)
    pipe.run(torch.from_numpy(S0).cuda(), seeds.rng_seed(presets.RNG_BASE, 0))
    torch.cuda.synchronize()
    pipe.capture()
    rows = providers.host_row_provider(p.graph())
    feats = providers.host_feat_provider(p)
    for b in (1, 2):
        S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
        rs = seeds.rng_seed(presets.RNG_BASE, b)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        ref = oracle.minibatch(rows, feats, S, p.fanouts, rs)
        for h in range(len(p.fanouts)):
            got, exp = pipe.result(h), ref["hops"][h]
            for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                assert np.array_equal(got[k], exp[k]), (b, h, k)
        assert np.array_equal(pipe.features(), ref["X"])
    assert dsm.device_error() == 0


@pytest.mark.slow
def test_papers100m_shaped_batch_bit_exact():
    """configs[2] shape on ONE GPU (111M nodes, ~3.2B CSR entries, 128 x fp32 = 57 GB of
    features; 83 GB of shards): one whole [15,10,5] batch of 1024 seeds, every array
    compared with the oracle (rows regenerated on the host for the touched nodes)."""
    p = presets.get("papers100m")
    free, _ = torch.cuda.mem_get_info()
    if free < 150e9:
        pytest.skip("needs a whole B200")
    dsm, info = loader.build_dsm(p, on_device=True)
    try:
        rp, col, _ = dsm.local_view()
        assert abs(int(rp[-1].item()) - p.target_e) / p.target_e < 0.03
        pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
        S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 7)
        rs = seeds.rng_seed(presets.RNG_BASE, 7)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        ref = oracle.minibatch(providers.host_row_provider(p.graph()), providers.host_feat_provider(p), S, p.fanouts, rs)
        for h in range(len(p.fanouts)):
            got, exp = pipe.result(h), ref["hops"][h]
            for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                assert np.array_equal(got[k], exp[k]), (h, k)
        assert np.array_equal(pipe.features(), ref["X"])
        assert dsm.device_error() == 0
    finally:
        dsm.destroy()


@pytest.mark.slow
def test_mag240m_shaped_graph_w4_virtual_ranks_bit_exact():
    """configs[4]'s graph at full size (244M nodes, ~3.4B CSR entries, fanout [25,15]) sharded
    over W=4 in-process virtual ranks on the one GPU (the config needs W >= 4).  The 768 x fp16
    table (375 GB) cannot fit one GPU, so the rows are narrowed to 16 x fp16 (32 B): the graph,
    the 4-way sharding, the G=32 lane groups of fanout 25 and the gather addressing are the
    config's; one batch per probed rank, every array compared with the oracle."""
    import threading

    from paper_conf_sc_yanglql22_b200.pipeline import required_keys
    from synth import gpu as sgpu

    p = presets.get("mag240m")
    W, FD, FDT = 4, 16, "fp16"
    free, _ = torch.cuda.mem_get_info()
    if free < 150e9:
        pytest.skip("needs a whole B200")
    spec = p.graph()
    shards = []
    for r in range(W):  # one shard at a time (generator temporaries are large)
        rp_r, col_r = sgpu.shard_csr_gpu(spec, r, W, torch.device("cuda", 0))
        shards.append((rp_r, col_r))
        torch.cuda.empty_cache()
    assert abs(sum(int(c.numel()) for _, c in shards) - p.target_e) / p.target_e < 0.03
    keys = required_keys(p.n, p.fanouts, p.seeds_per_batch)
    ag = pkg.ThreadAllgather(W)
    dsms, errs = [None] * W, []

    def create(r):
        try:
            dsms[r] = pkg.DSM(p.n, int(shards[r][1].numel()), FD, FDT, keys, rank=r, world_size=W, device=0,
                              allgather=ag.for_rank(r))
        except Exception as e:  # pragma: no cover
            errs.append(e)
    ths = [threading.Thread(target=create, args=(r,)) for r in range(W)]
    [t.start() for t in ths]
    [t.join() for t in ths]
    assert not errs, errs
    try:
        for r, d in enumerate(dsms):
            lrp, lcol, _ = d.local_view()
            lrp.copy_(shards[r][0])
            lcol.copy_(shards[r][1])
            sgpu.fill_dsm_features_gpu(d, presets.FEAT_SEED, r, W, FD, features.WG_DTYPE_CODE[FDT])
        del shards
        torch.cuda.synchronize()
        rows = providers.host_row_provider(spec)
        feats = providers.host_feat_provider(p, FD, FDT)
        for r in (0, 3):
            pipe = pkg.MiniBatchPipeline(dsms[r], p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
            b = next(iter(seeds.rank_batches(W, r, W)))
            S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
            rs = seeds.rng_seed(presets.RNG_BASE, b)
            pipe.run(torch.from_numpy(S).cuda(), rs)
            torch.cuda.synchronize()
            ref = oracle.minibatch(rows, feats, S, p.fanouts, rs)
            for h in range(len(p.fanouts)):
                got, exp = pipe.result(h), ref["hops"][h]
                for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                    assert np.array_equal(got[k], exp[k]), (r, h, k)
            assert np.array_equal(pipe.features(), ref["X"]), r
            assert dsms[r].device_error() == 0
            del pipe
    finally:
        ths = [threading.Thread(target=d.destroy) for d in dsms if d is not None]
        [t.start() for t in ths]
        [t.join() for t in ths]


def test_products_throughput_configuration_bit_exact(products):
    """The launch configuration of bench.py's throughput pass and e2e (8 batches in flight on DSM
    workspace forks and 8 streams, graph replay, gathers at the throughput occupancy, pinned-host
    seeds) at full products size: 16 batches, every array of every batch compared with the oracle."""
    p, dsm, _ = products
    depth, nb = 8, 16
    ld = pkg.MiniBatchLoader(dsm, p.fanouts, p.seeds_per_batch, depth=depth, with_pos=True, with_dup=True)
    assert all(pl.gather_occupancy == pkg.pipeline.THROUGHPUT_GATHER_OCCUPANCY for pl in ld.pipes)
    S = [seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 500 + b) for b in range(nb)]
    rs = [seeds.rng_seed(presets.RNG_BASE, 500 + b) for b in range(nb)]
    batches = [(torch.from_numpy(s).pin_memory(), r) for s, r in zip(S, rs)]
    rows = providers.host_row_provider(p.graph())
    feats = providers.host_feat_provider(p)
    seen = 0
    for pb in ld(batches):
        ref = oracle.minibatch(rows, feats, S[seen], p.fanouts, rs[seen])
        for h in range(len(p.fanouts)):
            got, exp = pb.hop(h), ref["hops"][h]
            for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                assert np.array_equal(got[k].cpu().numpy(), exp[k]), (seen, h, k)
        assert np.array_equal(pb.X.cpu().numpy(), ref["X"]), seen
        seen += 1
    assert seen == nb and ld.device_error() == 0
    ld.close()


@pytest.mark.slow
@pytest.mark.parametrize("placement", ["dsm", "csr-replicated"])
def test_products_w4_virtual_ranks_bit_exact(placement):
    """configs[1] at full size sharded over W=4 in-process virtual ranks on the one GPU, for the paper's
    placement (CSR and 400 B split feature rows row-sharded: most row_ptr / col_idx / feature reads go to
    other ranks' shards through the pointer table) and the CSR-replicated one (whole uint32 CSR per rank,
    features sharded): one batch on ranks 0 and 3, every array compared with the oracle."""
    import threading
    p = presets.get("products")
    W = 4
    flags = pkg.WG_DSM_CSR_REPLICATED if placement == "csr-replicated" else 0
    ag = pkg.ThreadAllgather(W)
    dsms, errs = [None] * W, []

    def create(r):
        try:
            dsms[r] = loader.build_dsm(p, rank=r, world=W, allgather=ag.for_rank(r), flags=flags)[0]
        except Exception as e:  # pragma: no cover
            errs.append(e)
    ths = [threading.Thread(target=create, args=(r,)) for r in range(W)]
    [t.start() for t in ths]
    [t.join() for t in ths]
    assert not errs, errs
    try:
        rows = providers.host_row_provider(p.graph())
        feats = providers.host_feat_provider(p)
        for r in (0, 3):
            if flags:
                assert dsms[r].local_view()[0].numel() == p.n + 1
            pipe = pkg.MiniBatchPipeline(dsms[r], p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
            b = next(iter(seeds.rank_batches(2 * W, r, W)))
            S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
            rs = seeds.rng_seed(presets.RNG_BASE, b)
            pipe.run(torch.from_numpy(S).cuda(), rs)
            torch.cuda.synchronize()
            ref = oracle.minibatch(rows, feats, S, p.fanouts, rs)
            for h in range(len(p.fanouts)):
                got, exp = pipe.result(h), ref["hops"][h]
                for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                    assert np.array_equal(got[k], exp[k]), (placement, r, h, k)
            assert np.array_equal(pipe.features(), ref["X"]), (placement, r)
            assert dsms[r].device_error() == 0
            del pipe
    finally:
        ths = [threading.Thread(target=d.destroy) for d in dsms if d is not None]
        [t.start() for t in ths]
        [t.join() for t in ths]
