"""Parity of the CUDA path (through the C ABI) with the CPU oracle: bit-exact
(tolerance 0) for sampled ids, positions, the sub-graph CSR, the unique/renumber
maps, the duplicate counts and the gathered feature bytes (BASELINE.json
north_star)."""

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import providers
from synth import features, graph, presets, seeds

from gpu_helpers import csr_from_rows, gpu_hop, gpu_sample_hop, gpu_unique, make_dsm, oracle_hop, oracle_sample_hop

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tiny():
    p = presets.get("tiny")
    rp, col = graph.csr(p.graph())
    return p, rp, col


def _check_batch(pipe, ref, fanouts):
    for h in range(len(fanouts)):
        got, exp = pipe.result(h), ref["hops"][h]
        for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
            assert np.array_equal(got[k], exp[k]), f"hop {h}: {k}"
    assert np.array_equal(pipe.features(), ref["X"])


@pytest.mark.parametrize("fused,incr", [(True, True), (False, True), (True, False)])
def test_tiny_pipeline_many_batches(tiny, fused, incr):
    """Config 1 (10k nodes, [10,5], 512 seeds): 20 batches, every array bit-exact, through
    the fused hop (wg_sample_hop) and through the separate ops (wg_sample_neighbors +
    wg_append_unique)."""
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True, fused=fused,
                                 incremental_gather=incr)
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    for b in range(20):
        S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
        rs = seeds.rng_seed(presets.RNG_BASE, b)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        ref = oracle.minibatch(rows, feats, S, p.fanouts, rs)
        _check_batch(pipe, ref, p.fanouts)
    assert dsm.device_error() == 0
    dsm.destroy()


@pytest.mark.parametrize("how", ["device", "host", "pinned", "packed"])
def test_pipeline_input_paths(tiny, how):
    """The batch inputs reach the captured graph through every set_inputs path -- device ids (D2D + 16 B
    H2D), host / pinned ids (packed into the pinned staging ring, one H2D), a packed device buffer
    (one D2D) -- with ragged seed counts, and every batch stays bit-exact."""
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    for b, cnt in enumerate([p.seeds_per_batch, 7, p.seeds_per_batch - 3, 1]):
        S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 40 + b)[:cnt]
        rs = seeds.rng_seed(presets.RNG_BASE, 40 + b)
        t = torch.from_numpy(S)
        if how == "device":
            pipe.set_inputs(t.cuda(), rs)
        elif how == "host":
            pipe.set_inputs(t, rs)
        elif how == "pinned":
            pipe.set_inputs(t.pin_memory(), rs)
        else:
            pipe.set_inputs_packed(pkg.pipeline.pack_inputs(S, rs, "cuda"))
        if pipe.graph is not None:
            pipe.graph.replay()
        else:
            pipe.enqueue()
        torch.cuda.synchronize()
        _check_batch(pipe, oracle.minibatch(rows, feats, S, p.fanouts, rs), p.fanouts)
        if b == 0:
            pipe.capture()
    assert dsm.device_error() == 0
    dsm.destroy()


def test_tiny_cuda_graph_replay(tiny):
    """The captured batch graph replays with new seeds / rng_seed and stays bit-exact."""
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
    S0 = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 0)
    pipe.run(torch.from_numpy(S0).cuda(), 1)
    torch.cuda.synchronize()
    pipe.capture()
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    for b in (3, 4, 5):
        n = 100 + 150 * (b - 3)      # fewer seeds than the capacity: device counts drive the graph
        S = seeds.seed_nodes(p.n, n, presets.SEED_BASE, b)
        rs = seeds.rng_seed(presets.RNG_BASE, b)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        _check_batch(pipe, oracle.minibatch(rows, feats, S, p.fanouts, rs), p.fanouts)
    assert dsm.device_error() == 0
    dsm.destroy()


def _edge_graph():
    """Degrees 0, 1, M-1, M, M+1 for several M, a 2^20 hub, and nodes whose rows
    are all each other (so a hop can add no new node)."""
    rng = np.random.default_rng(11)
    n = 5000
    rows = []
    for v in range(n):
        kind = v % 11
        d = [0, 1, 4, 5, 6, 9, 10, 11, 31, 32, 33][kind]
        rows.append(np.sort(rng.choice(n, size=d, replace=False)))
    hub = 4999
    rows[hub] = np.arange(1 << 20, dtype=np.int64) % n  # multi-edge hub row (positions are what is sampled)
    rows[0], rows[1], rows[2] = np.array([1, 2]), np.array([0, 2]), np.array([0, 1])
    return n, csr_from_rows(rows)


@pytest.mark.parametrize("M", [1, 5, 8, 9, 16, 17, 25, 32])
def test_sample_edge_cases(M):
    n, (rp, col) = _edge_graph()
    dsm = make_dsm(rp, col, max_keys=1 << 16)
    T = np.concatenate([np.arange(0, 200), [4999, 4998, 4997, n - 1 - 11]]).astype(np.int64)
    for hop, seed in ((0, 0x1234), (3, 0xFFFFFFFFFFFFFFFF)):
        g = gpu_hop(dsm, T, M, seed, hop)
        o = oracle_hop(rp, col, T, M, seed, hop)
        for a, b in zip(g, o):
            assert np.array_equal(a, b)
    # single target, and empty target list
    g = gpu_hop(dsm, np.array([4999]), M, 7, 1)
    assert np.array_equal(g[1], oracle_hop(rp, col, np.array([4999]), M, 7, 1)[1])
    rp0, nb0, _ = gpu_hop(dsm, np.zeros(0, np.int64), M, 7, 1)
    assert list(rp0) == [0] and len(nb0) == 0
    assert dsm.device_error() == 0
    dsm.destroy()


def test_sample_bad_ids_latch_error():
    n, (rp, col) = _edge_graph()
    dsm = make_dsm(rp, col)
    rp_g, nb, _ = gpu_hop(dsm, np.array([5, -1, n + 3, 7]), 4, 1, 0)
    assert dsm.device_error() & 0x1
    assert rp_g[2] - rp_g[1] == 0 and rp_g[3] - rp_g[2] == 0   # invalid ids read as degree 0
    dsm.destroy()


def test_append_unique_random_vs_oracle():
    n, (rp, col) = _edge_graph()
    dsm = make_dsm(rp, col, max_keys=1 << 20)
    rng = np.random.default_rng(5)
    for trial in range(30):
        pool = int(rng.integers(1, 4000))
        nT = int(rng.integers(0, min(pool, 3000) + 1))
        T = rng.choice(pool, size=nT, replace=False).astype(np.int64)
        nE = int(rng.integers(0, 200_000))
        # power-law-ish repeats (hubs) plus overlap with the targets
        nbrs = np.minimum((rng.random(nE) ** 3 * pool).astype(np.int64), pool - 1)
        U, sc, dup = gpu_unique(dsm, T, nbrs)
        Uo, sco, dupo = oracle.append_unique(T, nbrs)
        assert np.array_equal(U, Uo) and np.array_equal(sc, sco) and np.array_equal(dup, dupo)
    assert dsm.device_error() == 0
    # duplicate targets latch the error bit
    gpu_unique(dsm, np.array([3, 4, 3]), np.array([1, 2]))
    assert dsm.device_error() & 0x2
    # all neighbours are targets; empty neighbour list
    U, sc, _ = gpu_unique(dsm, np.array([40, 10, 30]), np.array([30, 40, 40]))
    assert list(U) == [40, 10, 30] and list(sc) == [2, 0, 0]
    U, sc, _ = gpu_unique(dsm, np.array([40, 10]), np.zeros(0, np.int64))
    assert list(U) == [40, 10]
    dsm.destroy()


@pytest.mark.parametrize("n_nbrs", [2_000_000, 2_200_000, 3_500_000])
def test_scan_prefix_forms_large(n_nbrs):
    """The flag scan takes the direct tile-prefix sum for <= WG_LB_DIRECT_MAX (1024) tiles of 2048 positions
    and the decoupled look-back above: append-unique calls on both sides of the boundary (977, 1075 and 1709
    tiles), and the standalone sampler's compaction scan (256 targets per tile) with 200k and 400k targets,
    all against the oracle."""
    n, (rp, col) = _edge_graph()
    dsm = make_dsm(rp, col, max_keys=4_000_000)
    rng = np.random.default_rng(n_nbrs)
    pool = n  # ids must be node ids; hub-heavy repeats (the scan sees every position)
    T = rng.choice(pool, size=3000, replace=False).astype(np.int64)
    nbrs = np.minimum((rng.random(n_nbrs) ** 2 * pool).astype(np.int64), pool - 1)
    U, sc, dup = gpu_unique(dsm, T, nbrs)
    Uo, sco, dupo = oracle.append_unique(T, nbrs)
    assert np.array_equal(U, Uo) and np.array_equal(sc, sco) and np.array_equal(dup, dupo)
    nT = 200_000 if n_nbrs < 3_000_000 else 400_000
    Ts = rng.integers(0, n, nT).astype(np.int64)
    got = gpu_hop(dsm, Ts, 3, 77, 1)
    exp = oracle_hop(rp, col, Ts, 3, 77, 1)
    for g, e in zip(got, exp):
        assert np.array_equal(g, e)
    assert dsm.device_error() == 0
    dsm.destroy()


@pytest.mark.parametrize("dim,dtype", [(4, "fp32"), (32, "fp32"), (100, "fp32"), (1024, "fp32"), (768, "fp16"),
                                       (3, "fp32"), (1, "fp16"), (7, "bf16"), (36, "fp32"), (56, "fp32"),
                                       (60, "fp32"), (200, "fp16"), (72, "bf16")])
def test_gather_rows(dim, dtype):
    """Row sizes 16 B .. 4 KB and non-multiples of 16 B, whole and split row layouts (144, 224, 240,
    400 B: body of whole 128 B lines + a tail of 16..112 B); repeated, sorted, reversed, empty id
    lists; dense and 32 B-pitched outputs (wg_gather_rows)."""
    n = 3000
    rp = np.zeros(n + 1, dtype=np.int64)
    feat = features.feature_bytes(presets.FEAT_SEED, np.arange(n), dim, dtype)
    dsm = make_dsm(rp, np.zeros(0, np.int64), feat, dim, dtype)
    rb = dsm.row_bytes
    if rb > 128 and rb % 128 and rb % 16 == 0:
        assert dsm.tail_pitch == rb % 128 and dsm.body_bytes == rb - rb % 128
    else:
        assert dsm.tail_pitch == 0 and dsm.body_bytes == rb
    # the shard holds exactly the generator's rows under either layout
    assert np.array_equal(dsm.read_local_rows(torch.arange(n, device="cuda")).cpu().numpy(), feat)
    rng = np.random.default_rng(dim)
    for ids in (rng.integers(0, n, 5000), np.arange(n), np.arange(n)[::-1], np.full(77, n - 1), np.zeros(0)):
        ids = np.ascontiguousarray(ids, dtype=np.int64)
        X = dsm.gather(torch.from_numpy(ids).cuda())
        torch.cuda.synchronize()
        exp = oracle.gather(feat, np.arange(n), ids)
        assert np.array_equal(X[:len(ids)].cpu().numpy(), exp)
        pitch = dsm.out_pitch()
        if pitch != rb and rb % 16 == 0 and len(ids):
            Xp = torch.zeros((len(ids), pitch), dtype=torch.uint8, device="cuda")
            begin = torch.zeros(1, dtype=torch.int64, device="cuda")
            end = torch.full((1,), len(ids), dtype=torch.int64, device="cuda")
            dsm.gather_rows(torch.from_numpy(ids).cuda(), len(ids), begin, end, Xp)
            torch.cuda.synchronize()
            assert np.array_equal(Xp[:, :rb].cpu().numpy(), exp)
        if rb % 32 == 16 and len(ids) > 4:
            # dense rows of R % 32 == 16 (32 B source pieces stored as 16 B halves for R >= 48, else the
            # 16 B-vector path): whole lists and row ranges starting / ending on odd rows; bytes outside the
            # range stay put
            for b, e in ((0, len(ids)), (1, len(ids) - 1), (3, 4), (2, len(ids) - 3)):
                Xd = torch.full((len(ids), rb), 0xCD, dtype=torch.uint8, device="cuda")
                be = torch.tensor([b, e], dtype=torch.int64, device="cuda")
                dsm.gather_rows(torch.from_numpy(ids).cuda(), len(ids), be[0:1], be[1:2], Xd)
                torch.cuda.synchronize()
                xd = Xd.cpu().numpy()
                assert np.array_equal(xd[b:e], exp[b:e]), (b, e)
                assert (xd[:b] == 0xCD).all() and (xd[e:] == 0xCD).all(), (b, e)
    assert dsm.device_error() == 0
    dsm.destroy()


def test_feat_whole_rows_flag():
    """WG_DSM_WHOLE_ROWS (whole rows at a 64 B pitch instead of the split body + tail layout)
    gathers the same bytes."""
    for dim, dtype in ((100, "fp32"), (36, "fp32"), (200, "fp16")):
        n = 4000
        rp = np.zeros(n + 1, dtype=np.int64)
        feat = features.feature_bytes(presets.FEAT_SEED, np.arange(n), dim, dtype)
        dsm = make_dsm(rp, np.zeros(0, np.int64), feat, dim, dtype, flags=pkg.WG_DSM_WHOLE_ROWS)
        assert dsm.tail_pitch == 0 and dsm.body_bytes == dsm.row_bytes
        ids = np.random.default_rng(dim).integers(0, n, 6000).astype(np.int64)
        X = dsm.gather(torch.from_numpy(ids).cuda())
        torch.cuda.synchronize()
        assert np.array_equal(X.cpu().numpy(), oracle.gather(feat, np.arange(n), ids)), (dim, dtype)
        dsm.destroy()


def test_pipeline_dense_x_400b_rows():
    """A pipeline with a dense X (pitch = the 400 B row, 32 B source pieces stored as 16 B halves; incremental
    gathers start on odd rows) is bit-exact, and so is the 32 B-pitched X (416 B)."""
    n, dim = 3000, 100
    rng = np.random.default_rng(5)
    rows = [np.unique(rng.integers(0, n, rng.integers(0, 40))) for _ in range(n)]
    rows = [r[r != v] for v, r in enumerate(rows)]
    g_rp, g_col = csr_from_rows(rows)
    feat = features.feature_bytes(presets.FEAT_SEED, np.arange(n), dim, "fp32")
    dsm = make_dsm(g_rp, g_col, feat, dim, "fp32", max_keys=1 << 16)
    assert dsm.out_pitch() == 416
    rowsf = providers.host_row_provider(None, g_rp, g_col)

    def feats(ids):
        u = np.unique(np.asarray(ids, dtype=np.int64))
        return u, features.feature_bytes(presets.FEAT_SEED, u, dim, "fp32")
    for xp in (dim * 4, 416):
        pipe = pkg.MiniBatchPipeline(dsm, [7, 4], 101, with_pos=True, with_dup=True, x_pitch=xp)
        for b in range(6):
            S = np.random.default_rng(100 + b).choice(n, 101 - 2 * b, replace=False).astype(np.int64)
            pipe.run(torch.from_numpy(S).cuda(), 77 + b)
            torch.cuda.synchronize()
            _check_batch(pipe, oracle.minibatch(rowsf, feats, S, [7, 4], 77 + b), [7, 4])
            if b == 0:
                pipe.capture()
    assert dsm.device_error() == 0
    dsm.destroy()


def test_determinism_two_runs(tiny):
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
    S = torch.from_numpy(seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 9)).cuda()
    outs = []
    for _ in range(2):
        pipe.run(S, 99)
        torch.cuda.synchronize()
        outs.append([pipe.result(h) for h in range(2)] + [pipe.features()])
    for a, b in zip(outs[0][:2], outs[1][:2]):
        for k in a:
            assert np.array_equal(a[k], b[k])
    assert np.array_equal(outs[0][2], outs[1][2])
    dsm.destroy()


def test_fork_concurrent_streams(tiny):
    """wg_dsm_fork: two pipelines on the same shards, different workspaces, running
    concurrently on two streams, both bit-exact."""
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False)
    child = dsm.fork()
    pipes = [pkg.MiniBatchPipeline(h, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
             for h in (dsm, child)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    for rnd in range(3):
        Ss, rss = [], []
        for j in range(2):
            b = 100 + 2 * rnd + j
            S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
            rs = seeds.rng_seed(presets.RNG_BASE, b)
            Ss.append(S)
            rss.append(rs)
            st = streams[j]
            st.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(st):
                pipes[j].set_inputs(torch.from_numpy(S).cuda(), rs, stream=st)
                pipes[j].enqueue(st)
        torch.cuda.synchronize()
        for j in range(2):
            _check_batch(pipes[j], oracle.minibatch(rows, feats, Ss[j], p.fanouts, rss[j]), p.fanouts)
    assert dsm.device_error() == 0 and child.device_error() == 0
    with pytest.raises(pkg.WgError):
        dsm.destroy()            # forks first
    child.destroy()
    dsm.destroy()


@pytest.mark.parametrize("M", [33, 64, 100, 257, 1024])
def test_sample_large_fanout_block_kernel(M):
    """fanout > 32: block per target running Algorithm 1 with a block bitonic sort (NEXT #4)."""
    rng = np.random.default_rng(M)
    n = 3000
    degs = [0, 1, 32, 33, M - 1, M, M + 1, 2 * M, 5000]
    rows = [np.sort(rng.choice(n, size=min(degs[v % len(degs)], n), replace=False)) if degs[v % len(degs)] <= n
            else rng.integers(0, n, degs[v % len(degs)]) for v in range(n)]
    rp, col = csr_from_rows(rows)
    dsm = make_dsm(rp, col, max_keys=1 << 20)
    T = np.arange(0, 400, dtype=np.int64)
    for hop, seed in ((0, 99), (2, 0xDEADBEEF12345678)):
        g = gpu_hop(dsm, T, M, seed, hop)
        o = oracle_hop(rp, col, T, M, seed, hop)
        for a, b in zip(g, o):
            assert np.array_equal(a, b)
    assert dsm.device_error() == 0
    dsm.destroy()


def test_pipeline_five_hops_fused(tiny):
    """More hops than the workspace's ring of 4 scan buffers: the fused pipeline joins the relabel side
    stream before hop 4 reuses hop 0's buffer, so every hop's sub_col / dup stays exact (captured graph)."""
    p, rp, col = tiny
    fan = [4, 3, 2, 2, 2]
    dsm, _ = loader.build_dsm(p, on_device=False, max_seeds=64, extra_keys=pkg.required_keys(p.n, fan, 64))
    pipe = pkg.MiniBatchPipeline(dsm, fan, 64, with_pos=True, with_dup=True)
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    for b in range(4):
        S = seeds.seed_nodes(p.n, 64, presets.SEED_BASE, 700 + b)
        rs = seeds.rng_seed(presets.RNG_BASE, 700 + b)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        _check_batch(pipe, oracle.minibatch(rows, feats, S, fan, rs), fan)
        if b == 0:
            pipe.capture()
    assert dsm.device_error() == 0
    dsm.destroy()


@pytest.mark.parametrize("col32", [False, True])
def test_pipeline_large_fanout(tiny, col32):
    """Fan-outs above 32 (the block sampler), int64 and uint32 (WG_DSM_COL32) col_idx."""
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False, max_seeds=64, extra_keys=64 * 60 * 41 + 64 * 60, col32=col32)
    fan = [60, 40]
    pipe = pkg.MiniBatchPipeline(dsm, fan, 64, with_pos=True, with_dup=True)
    S = seeds.seed_nodes(p.n, 64, presets.SEED_BASE, 3)
    rs = seeds.rng_seed(presets.RNG_BASE, 3)
    pipe.run(torch.from_numpy(S).cuda(), rs)
    torch.cuda.synchronize()
    ref = oracle.minibatch(providers.host_row_provider(p.graph(), rp, col), providers.host_feat_provider(p), S, fan, rs)
    _check_batch(pipe, ref, fan)
    assert dsm.device_error() == 0
    dsm.destroy()


def test_spmm_mean_forward_backward_vs_oracle(tiny):
    """NEXT #2: g-SpMM mean aggregation on the last hop's sub-graph CSR with the gathered
    features (float32), forward and backward (atomics + duplicate-count stores) against the
    float64 oracle; fp32 tolerance: <= 16-term sums in forward, atomics order in backward."""
    from paper_conf_sc_yanglql22_b200 import layers
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_dup=True)
    S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 11)
    pipe.run(torch.from_numpy(S).cuda(), seeds.rng_seed(presets.RNG_BASE, 11))
    torch.cuda.synchronize()
    h = pipe.result(1)
    nT = len(pipe.result(0)["unique"])
    U = len(h["unique"])
    X = torch.from_numpy(pipe.features().view(np.float32).reshape(U, p.feat_dim).copy()).cuda()
    row_ptr = torch.from_numpy(h["row_ptr"]).cuda()
    sub_col = torch.from_numpy(h["sub_col"]).cuda()
    dup = torch.from_numpy(h["dup"]).cuda()
    Y = layers.spmm_mean_forward(row_ptr, sub_col, X)
    Yo = oracle.spmm_mean_forward(h["row_ptr"], h["sub_col"], X.cpu().double().numpy())
    assert Y.shape == (nT, p.feat_dim)
    assert np.allclose(Y.cpu().numpy(), Yo, rtol=0, atol=1e-5)
    dY = torch.from_numpy(np.random.default_rng(1).uniform(-1, 1, (nT, p.feat_dim)).astype(np.float32)).cuda()
    dX = layers.spmm_mean_backward(row_ptr, sub_col, dup, dY, U)
    dX_nodup = layers.spmm_mean_backward(row_ptr, sub_col, None, dY, U)
    dXo = oracle.spmm_mean_backward(h["row_ptr"], h["sub_col"], dY.cpu().double().numpy(), U)
    assert np.allclose(dX.cpu().numpy(), dXo, rtol=1e-5, atol=1e-5)
    assert np.allclose(dX.cpu().numpy(), dX_nodup.cpu().numpy(), rtol=1e-5, atol=1e-5)
    # autograd wrapper
    Xg = X.clone().requires_grad_(True)
    out = layers.SpMMMean.apply(Xg, row_ptr, sub_col, dup)
    (out * dY).sum().backward()
    assert np.allclose(Xg.grad.cpu().numpy(), dXo, rtol=1e-5, atol=1e-5)
    # the pipeline's untrimmed buffers with the device row count (the previous hop's num_unique)
    b = pipe.hops[1]
    Xg2 = X.clone().requires_grad_(True)
    out2 = layers.SpMMMean.apply(Xg2, b["row_ptr"], b["sub_col"], b["dup"], pipe.hops[0]["num_unique"])
    assert np.allclose(out2[:nT].detach().cpu().numpy(), Yo, rtol=0, atol=1e-5)
    assert not out2[nT:].any()
    dYp = torch.zeros_like(out2)
    dYp[:nT] = dY
    (out2 * dYp).sum().backward()
    assert np.allclose(Xg2.grad.cpu().numpy(), dXo, rtol=1e-5, atol=1e-5)
    # an out-of-range sub-graph id (the -1 of an invalid id) is skipped, never dereferenced
    bad = sub_col.clone()
    bad[0] = -1
    bad[1] = U + 5
    Yb = layers.spmm_mean_forward(row_ptr, bad, X)
    dXb = layers.spmm_mean_backward(row_ptr, bad, dup, dY, U)
    torch.cuda.synchronize()
    assert torch.isfinite(Yb).all() and torch.isfinite(dXb).all()
    dsm.destroy()


def test_distributed_memory_gather_w1():
    """NEXT #1 baseline (NCCL-style five-step gather) equals the P2P gather byte for byte."""
    from paper_conf_sc_yanglql22_b200.nccl_gather import DistributedGather
    n, dim = 5000, 100
    rp = np.zeros(n + 1, dtype=np.int64)
    feat = features.feature_bytes(presets.FEAT_SEED, np.arange(n), dim, "fp32")
    dsm = make_dsm(rp, np.zeros(0, np.int64), feat, dim, "fp32")
    ids = torch.from_numpy(np.random.default_rng(3).integers(0, n, 20000)).cuda()
    b = DistributedGather(dsm).gather(ids)
    torch.cuda.synchronize()
    exp = oracle.gather(feat, np.arange(n), ids.cpu().numpy())   # the closed-form rows, not the P2P path
    assert np.array_equal(b[:20000].cpu().numpy(), exp)
    assert dsm.device_error() == 0
    dsm.destroy()


def test_pipeline_degenerate_batches(tiny):
    """Empty seed list, a single seed, seeds whose rows are empty: device counts of 0 flow
    through every kernel of the captured graph."""
    p, rp, col = tiny
    n = 64
    rows = [[] for _ in range(n)]
    rows[5] = [6, 7]
    rows[6] = [5]
    g_rp, g_col = csr_from_rows(rows)
    feat = features.feature_bytes(presets.FEAT_SEED, np.arange(n), 8, "fp32")
    dsm = make_dsm(g_rp, g_col, feat, 8, "fp32", max_keys=4096)
    pipe = pkg.MiniBatchPipeline(dsm, [3, 2], 16, with_pos=True, with_dup=True)
    rowsf = providers.host_row_provider(None, g_rp, g_col)

    def feats(ids):
        u = np.unique(np.asarray(ids, dtype=np.int64))
        return u, features.feature_bytes(presets.FEAT_SEED, u, 8, "fp32")
    pipe.run(torch.from_numpy(np.array([1], np.int64)).cuda(), 3)
    torch.cuda.synchronize()
    pipe.capture()
    for S in (np.zeros(0, np.int64), np.array([0, 1, 2], np.int64), np.array([5], np.int64), np.array([9, 5, 6], np.int64)):
        pipe.run(torch.from_numpy(S).cuda() if len(S) else torch.zeros(0, dtype=torch.int64, device="cuda"), 11)
        torch.cuda.synchronize()
        ref = oracle.minibatch(rowsf, feats, S, [3, 2], 11)
        _check_batch(pipe, ref, [3, 2])
    assert dsm.device_error() == 0
    dsm.destroy()


def test_epoch_exhaustion_and_reset():
    """The wide table's epoch space: near its end an op latches WG_DEVERR_EPOCH;
    wg_dsm_reset_workspace restores correct operation (test hook wg_dsm_debug_set_epoch)."""
    T = np.array([4, 9], np.int64)
    nb = np.array([1, 4, 1, 7], np.int64)
    dsm = make_dsm(np.zeros(11, np.int64), np.zeros(0, np.int64), max_keys=64, flags=pkg.WG_DSM_WIDE_HASH)
    dsm.debug_set_epoch((1 << 23) - 3)
    U, sc, dup = gpu_unique(dsm, T, nb)          # uses epoch EPOCH_MAX-2 -> bumps to EPOCH_MAX-1
    assert list(U) == [4, 9, 1, 7] and dsm.device_error() == 0
    gpu_unique(dsm, T, nb)                       # epoch + 1 would reach EPOCH_MAX: latched
    assert dsm.device_error() & 0x10
    dsm.reset_workspace()
    torch.cuda.synchronize()
    for _ in range(3):
        U, sc, dup = gpu_unique(dsm, T, nb)
        Uo, sco, dupo = oracle.append_unique(T, nb)
        assert np.array_equal(U, Uo) and np.array_equal(sc, sco) and np.array_equal(dup, dupo)
    assert dsm.device_error() == 0
    with pytest.raises(pkg.WgError):
        dsm.debug_set_epoch(0)
    dsm.destroy()


@pytest.mark.parametrize("fmt", ["direct", "compact"])
def test_compact_table_epoch_cycles(tiny, fmt):
    """The compact 8 B hash table and the direct tables cycle through 255 epochs and are cleared when
    a cycle restarts (compact: by the fused hop's sampler, or before a standalone insert; direct: the
    op at epoch e clears the idle table of epoch e+1): 140 tiny batches (280 fused hops, more than a
    whole cycle, starting just before a restart) and standalone append-unique calls across a
    restart, all bit-exact against the oracle."""
    fl = 0 if fmt == "direct" else pkg.WG_DSM_HASHED
    want = pkg.WG_UNIQUE_DIRECT if fmt == "direct" else pkg.WG_UNIQUE_COMPACT
    p, rp, col = tiny
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    dsm, _ = loader.build_dsm(p, on_device=False, flags=fl)
    assert dsm.unique_format() == want
    dsm.debug_set_epoch(250)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
    pipe.run(torch.from_numpy(seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 0)).cuda(), 5)
    pipe.capture()
    for b in range(140):
        S = seeds.seed_nodes(p.n, p.seeds_per_batch - (b % 5) * 11, presets.SEED_BASE, 1000 + b)
        rs = seeds.rng_seed(presets.RNG_BASE, 1000 + b)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        _check_batch(pipe, oracle.minibatch(rows, feats, S, p.fanouts, rs), p.fanouts)
    assert dsm.device_error() == 0
    dsm.destroy()
    rng = np.random.default_rng(3)
    d2 = make_dsm(np.zeros(2001, np.int64), np.zeros(0, np.int64), max_keys=4096, flags=fl)
    assert d2.unique_format() == want
    d2.debug_set_epoch(250)
    for i in range(300):
        if i == 150:   # the next cycle restart (direct: back to the first table)
            d2.debug_set_epoch(508)
        if i == 200:   # the counter's wrap (modulo 2 x 255 epochs: cycle parity and tags continue)
            d2.debug_set_epoch(2 * 255 * 2048 - 3)
        T = rng.choice(2000, 40, replace=False).astype(np.int64)
        nb = rng.integers(0, 2000, 600).astype(np.int64)
        U, sc, dup = gpu_unique(d2, T, nb)
        Uo, sco, dupo = oracle.append_unique(T, nb)
        assert np.array_equal(U, Uo) and np.array_equal(sc, sco) and np.array_equal(dup, dupo), i
    assert d2.device_error() == 0
    d2.destroy()


def test_gather_occupancy_setting(tiny):
    """wg_dsm_set_gather_occupancy changes only the launch shape: every occupancy gathers the same
    bytes, directly and through a captured pipeline graph (values restored after enqueue)."""
    p, rp, col = tiny
    dsm, _ = loader.build_dsm(p, on_device=False)
    S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 5)
    rs = seeds.rng_seed(presets.RNG_BASE, 5)
    ref = oracle.minibatch(providers.host_row_provider(p.graph(), rp, col), providers.host_feat_provider(p), S,
                           p.fanouts, rs)
    for occ in (1, 2, 3, 0):
        pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, gather_occupancy=occ)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        pipe.capture()
        pipe.X.zero_()
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        assert dsm.gather_occupancy == 0
        assert np.array_equal(pipe.features(), ref["X"]), occ
    with pytest.raises(pkg.WgError):
        dsm.set_gather_occupancy(-1)
    assert dsm.device_error() == 0
    dsm.destroy()


@pytest.mark.parametrize("flags", ["WG_DSM_WIDE_HASH", "WG_DSM_PAD64", "WG_DSM_WIDE_HASH|WG_DSM_PAD64", "COL64",
                                   "COL64|WG_DSM_PAD64", "WG_DSM_HASHED", "WG_DSM_HASHED|WG_DSM_PAD64"])
def test_table_and_slot_formats(tiny, flags):
    """The non-default hash-table / padded-slot / column formats (16 B wide slots claimed with one 128-bit
    CAS, int64 padded sampler slots, int64 col_idx instead of the loader's default uint32) stay bit-exact: 12 tiny batches through the fused
    pipeline and hub-heavy standalone append-unique calls."""
    fl = 0
    for f in flags.split("|"):
        fl |= getattr(pkg, f) if f != "COL64" else 0
    p, rp, col = tiny
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    dsm, _ = loader.build_dsm(p, on_device=False, flags=fl, col32="COL64" not in flags)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
    for b in range(12):
        S = seeds.seed_nodes(p.n, p.seeds_per_batch - b * 7, presets.SEED_BASE, 300 + b)
        rs = seeds.rng_seed(presets.RNG_BASE, 300 + b)
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        _check_batch(pipe, oracle.minibatch(rows, feats, S, p.fanouts, rs), p.fanouts)
    assert dsm.device_error() == 0
    dsm.destroy()
    rng = np.random.default_rng(11)
    d2 = make_dsm(np.zeros(5001, np.int64), np.zeros(0, np.int64), max_keys=1 << 16, flags=fl)
    for i in range(20):
        T = rng.choice(5000, 300, replace=False).astype(np.int64)
        nb = np.minimum((rng.pareto(1.2, 20000) * 3).astype(np.int64), 4999)   # hub-heavy
        U, sc, dup = gpu_unique(d2, T, nb)
        Uo, sco, dupo = oracle.append_unique(T, nb)
        assert np.array_equal(U, Uo) and np.array_equal(sc, sco) and np.array_equal(dup, dupo), i
    assert d2.device_error() == 0
    d2.destroy()


def test_unique_format_selection(tiny):
    """wg_dsm_unique_format: the direct table for small graphs, the compact hash with WG_DSM_HASHED, the
    wide hash with WG_DSM_WIDE_HASH; and a graph too large for the direct table (num_nodes > 2^24) is
    hashed."""
    p, rp, col = tiny
    for fl, want in ((0, pkg.WG_UNIQUE_DIRECT), (pkg.WG_DSM_HASHED, pkg.WG_UNIQUE_COMPACT),
                     (pkg.WG_DSM_WIDE_HASH, pkg.WG_UNIQUE_WIDE),
                     (pkg.WG_DSM_WIDE_HASH | pkg.WG_DSM_HASHED, pkg.WG_UNIQUE_WIDE)):
        dsm = make_dsm(np.zeros(101, np.int64), np.zeros(0, np.int64), max_keys=64, flags=fl)
        assert dsm.unique_format() == want, fl
        dsm.destroy()
    big = make_dsm(np.zeros((1 << 24) + 2, np.int64), np.zeros(0, np.int64), max_keys=64)
    assert big.unique_format() == pkg.WG_UNIQUE_COMPACT
    big.destroy()
    # at the boundary (2^24 nodes) the direct table is used; ids near the top of the range round-trip
    n = 1 << 24
    rp = np.zeros(n + 1, np.int64)
    hub = n - 1
    rp[hub + 1:] = 40  # node n-1 has 40 neighbours, all near the top of the id range (and itself excluded)
    col = (n - 2 - np.arange(40, dtype=np.int64) * 7919 % (n - 1))
    edge = make_dsm(rp, col, max_keys=1 << 12)
    assert edge.unique_format() == pkg.WG_UNIQUE_DIRECT
    T = np.array([hub, 5, n - 2], np.int64)
    got = gpu_sample_hop(edge, T, 10, 99, 1)
    ref = oracle_sample_hop(rp, col, T, 10, 99, 1)
    for g, r in zip(got, ref):
        assert np.array_equal(g, r)
    assert edge.device_error() == 0
    edge.destroy()


@pytest.mark.parametrize("fl", [0, "WG_DSM_HASHED"])
def test_direct_fused_hop_duplicate_and_bad_targets(fl):
    """Fused hop (the direct table's sampler-side inserts): duplicate targets latch WG_DEVERR_DUP_TARGET
    (A8), out-of-range targets and neighbours latch WG_DEVERR_ID_RANGE (B3), and a valid batch after
    them is bit-exact again."""
    flags = 0 if fl == 0 else getattr(pkg, fl)
    n, (rp, col) = _edge_graph()
    dsm = make_dsm(rp, col, max_keys=1 << 16, flags=flags)
    T = np.array([5, 9, 5, 7], np.int64)
    gpu_sample_hop(dsm, T, 4, 1, 0)
    assert dsm.device_error() & 0x2               # (device_error clears the word)
    gpu_sample_hop(dsm, np.array([5, n + 9, 7], np.int64), 4, 1, 0)
    assert dsm.device_error() & 0x1
    T = np.array([5, 9, 7, 11, 4999, 0, 1, 2], np.int64)
    got = gpu_sample_hop(dsm, T, 4, 3, 2)
    ref = oracle_sample_hop(rp, col, T, 4, 3, 2)
    for g, r in zip(got, ref):
        assert np.array_equal(g, r)
    assert dsm.device_error() == 0
    dsm.destroy()


@pytest.mark.parametrize("dim", [4, 100, 132, 260])
def test_spmm_mean_row_lengths_and_widths(dim):
    """g-SpMM forward / backward on a hand-made CSR whose rows have 0, 1, 5, 31, 32, 33, 40 and 300 edges
    (the forward's lane-held ids cover 32 edges, the rest come from a loop) and feature widths of 1 to 65
    float4 slices (more than one slice per lane), with repeated columns and invalid ids, against the fp64
    oracle (fp32 tolerance)."""
    from paper_conf_sc_yanglql22_b200 import layers
    rng = np.random.default_rng(dim)
    lens = [0, 1, 5, 31, 32, 33, 40, 300, 7, 0, 64]
    n_x = 500
    rows = [rng.integers(0, n_x, k) for k in lens]
    rp, col = csr_from_rows(rows)
    X = rng.uniform(-1, 1, (n_x, dim)).astype(np.float32)
    dY = rng.uniform(-1, 1, (len(lens), dim)).astype(np.float32)
    rp_t, col_t = torch.from_numpy(rp).cuda(), torch.from_numpy(col.astype(np.int32)).cuda()
    Y = layers.spmm_mean_forward(rp_t, col_t, torch.from_numpy(X).cuda())
    assert np.allclose(Y.cpu().numpy(), oracle.spmm_mean_forward(rp, col, X.astype(np.float64)), rtol=0, atol=2e-5)
    dup = np.bincount(col, minlength=n_x).astype(np.int32)
    dX = layers.spmm_mean_backward(rp_t, col_t, torch.from_numpy(dup).cuda(), torch.from_numpy(dY).cuda(), n_x)
    assert np.allclose(dX.cpu().numpy(), oracle.spmm_mean_backward(rp, col, dY.astype(np.float64), n_x),
                       rtol=1e-5, atol=2e-5)
    bad = col_t.clone()
    bad[3] = -1
    bad[50] = n_x + 7
    Yb = layers.spmm_mean_forward(rp_t, bad, torch.from_numpy(X).cuda())
    keep = np.ones(len(col), bool)
    keep[[3, 50]] = False
    # skipped edges still count in the mean's denominator (the row's degree)
    ref = np.zeros((len(lens), dim))
    for t in range(len(lens)):
        b, e = rp[t], rp[t + 1]
        idx = [k for k in range(b, e) if keep[k]]
        if e > b:
            ref[t] = X[col[idx]].astype(np.float64).sum(0) / (e - b)
    assert np.allclose(Yb.cpu().numpy(), ref, rtol=0, atol=2e-5)


@pytest.mark.parametrize("fl", [0, "WG_DSM_HASHED", "WG_DSM_WIDE_HASH"])
def test_fused_hop_invalid_neighbour_ids(fl):
    """A col_idx entry outside [0, n) (a corrupt graph, reading B3) through the fused hop of every key-table
    format: WG_DEVERR_ID_RANGE is latched, the sample stays in the CSR with the invalid id, is never
    numbered (sub_col -1, not in U), and every valid neighbour is numbered exactly as the oracle numbers the
    neighbour list without it."""
    flags = 0 if fl == 0 else getattr(pkg, fl)
    n = 50
    rows = [np.array([(v + 1) % n, (v + 7) % n], np.int64) for v in range(n)]
    rows[3] = np.array([4, n + 11, 9], np.int64)      # one invalid entry (int64 col storage)
    rp, col = csr_from_rows(rows)
    dsm = make_dsm(rp, col, max_keys=1 << 10, flags=flags)
    T = np.array([3, 10, 20], np.int64)
    rp_g, nb, pos, U, sc, dup = gpu_sample_hop(dsm, T, 8, 5, 0)   # fanout >= degree: whole rows, CSR order
    assert dsm.device_error() & 0x1
    assert list(rp_g) == [0, 3, 5, 7] and list(nb[:3]) == [4, n + 11, 9]
    assert sc[1] == -1 and (n + 11) not in set(U.tolist())
    keep = np.array([k for k in range(len(nb)) if k != 1])
    Uo, sco, dupo = oracle.append_unique(T, nb[keep])
    assert np.array_equal(U, Uo) and np.array_equal(sc[keep], sco)
    dsm.destroy()
