"""Properties of the seeded input generators (CPU only)."""

import numpy as np

from synth import features, graph, hashing, presets, seeds


def test_splitmix_reference_values():
    # splitmix64 from seed 0: first outputs of the reference generator
    # (Vigna, "splitmix64.c": x += golden; mix) are e220a8397b1dcdaf, 6e789e6aa1b965f4
    assert int(hashing.splitmix64(np.array([0], np.uint64))[0]) == 0xE220A8397B1DCDAF
    assert int(hashing.splitmix64(np.array([0x9E3779B97F4A7C15], np.uint64))[0]) == 0x6E789E6AA1B965F4
    assert hashing.splitmix64_int(0) == 0xE220A8397B1DCDAF


def test_rows_sorted_unique_no_self_loops_and_row_local():
    spec = presets.get("tiny").graph()
    rp, col = graph.csr(spec)
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0)
    for v in range(0, spec.n, 97):
        r = col[rp[v]:rp[v + 1]]
        assert np.all(np.diff(r) > 0) and not np.any(r == v)
        assert np.all((r >= 0) & (r < spec.n))
    assert np.all(np.diff(rp) <= graph.raw_degree(spec, np.arange(spec.n)))
    # row-locality: rows of an arbitrary subset (with repeats) equal the CSR rows
    sub = np.array([5, 9999, 0, 5, 1234], dtype=np.int64)
    ptr, c = graph.rows(spec, sub)
    for k, v in enumerate(sub):
        assert np.array_equal(c[ptr[k]:ptr[k + 1]], col[rp[v]:rp[v + 1]])
    # size lands near the configured target (calibrated d_min)
    assert abs(rp[-1] - 200_000) / 200_000 < 0.02


def test_power_law_shape():
    spec = presets.get("tiny").graph()
    rp, col = graph.csr(spec)
    indeg = np.bincount(col, minlength=spec.n)
    # low ids are in-degree hubs (gamma = 2.5)
    assert indeg[:100].mean() > 10 * indeg[-5000:].mean()
    assert np.diff(rp).max() > 50 * np.diff(rp).mean()


def test_feature_bits_range():
    for dtype in ("fp32", "fp16", "bf16"):
        b = features.feature_bits(7, np.arange(50), 33, dtype)
        if dtype == "fp32":
            v = b.view(np.float32)
        elif dtype == "fp16":
            v = b.view(np.float16).astype(np.float32)
        else:
            v = (b.astype(np.uint32) << 16).view(np.float32)
        assert np.all((v >= 1.0) & (v < 2.0))


def test_seed_nodes_unique_and_rank_batches():
    s = seeds.seed_nodes(1000, 512, 1, 3)
    assert len(np.unique(s)) == 512 and s.dtype == np.int64
    assert np.array_equal(s, seeds.seed_nodes(1000, 512, 1, 3))
    assert seeds.rank_batches(10, 1, 4) == [1, 5, 9]
    assert seeds.rng_seed(5, 2) != seeds.rng_seed(5, 3)


def test_shard_rows():
    assert list(graph.shard_rows(10, 1, 4)) == [1, 5, 9]
    assert sum(len(graph.shard_rows(11, r, 3)) for r in range(3)) == 11


def test_native_host_generator_matches_numpy():
    for name in ("tiny", "products", "papers100m", "mag240m"):
        spec = presets.get(name).graph()
        rng = np.random.default_rng(1)
        v = np.concatenate([[0, 1, spec.n - 1], rng.integers(0, spec.n, 300)]).astype(np.int64)
        p1, c1 = graph.rows(spec, v)
        p2, c2 = graph.rows_native(spec, v)
        assert np.array_equal(p1, p2) and np.array_equal(c1, c2), name


def test_native_features_match_numpy():
    v = np.array([0, 5, 2**33 + 7, 123456789], dtype=np.int64)
    for dtype, dim in (("fp32", 100), ("fp16", 768), ("bf16", 3)):
        assert np.array_equal(features.feature_bytes(9, v, dim, dtype), features.feature_bytes_native(9, v, dim, dtype))
