"""Pins of the CPU oracle against what the paper and the mathematics fix
(CPU only).  Each test names the oracle function it pins and the source of the
expected values; none of them re-derives an expected value by calling the
function under test with the same formula."""

import itertools
import math
import os

import numpy as np
import pytest
from scipy import stats

import oracle
from synth import features, graph, presets

from conftest import GOLDEN


def _read_golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line)
    return rows


# ---------------------------------------------------------------- Philox / draws
def test_philox_known_answers():
    """orc_philox4x32_10 vs the Random123 known-answer vectors."""
    for line in _read_golden("philox4x32_10_kat.txt"):
        w = [int(x, 16) for x in line.split()]
        out = oracle.philox4x32_10(w[0:4], w[4:6])
        assert [int(x) for x in out] == w[6:10], line


def test_draw_closed_form_and_range():
    """orc_draw = floor(x*(N-i)/2^32) on the KAT-pinned Philox word (A3), and r <= N-1-i (A2)."""
    rng = np.random.default_rng(1)
    for _ in range(300):
        seed = int(rng.integers(0, 2**63)) * 2 + int(rng.integers(0, 2))
        hop = int(rng.integers(0, 4))
        node = int(rng.integers(0, 2**40))
        N = int(rng.integers(2, 2**31))
        i = int(rng.integers(0, min(N, 40)))
        x = oracle.philox4x32_10([i >> 2, hop, node & 0xFFFFFFFF, node >> 32],
                                 [seed & 0xFFFFFFFF, seed >> 32])[i & 3]
        r = oracle.draw(seed, hop, node, i, N)
        assert r == (int(x) * (N - i)) >> 32
        assert 0 <= r <= N - 1 - i
    # extreme words: x = 0 -> 0, x = 2^32-1 -> N-1-i (inclusive upper end reachable)
    assert ((2**32 - 1) * 7) >> 32 == 6


# ---------------------------------------------------------------- Algorithm 1
def fisher_yates_partial(N, M, r):
    """Textbook sequential partial Fisher-Yates on a virtual array A[k] = k:
    step i outputs A[r_i] then moves A[N-1-i] into slot r_i (Durstenfeld 1964)."""
    A = list(range(N))
    out = []
    for i in range(M):
        out.append(A[r[i]])
        A[r[i]] = A[N - 1 - i]
    return out


def test_algorithm1_equals_fisher_yates_exhaustive():
    """orc_algorithm1 == sequential Fisher-Yates for every N <= 7, M < N and every
    draw vector (10,151 cases), and r -> res is a bijection onto the ordered
    M-permutations of [0, N) (hence exactly uniform for uniform r)."""
    cases = 0
    for N in range(2, 8):
        for M in range(1, N):
            seen = set()
            for r in itertools.product(*[range(N - i) for i in range(M)]):
                res = [int(x) for x in oracle.algorithm1(M, N, list(r))]
                assert res == fisher_yates_partial(N, M, r), (N, M, r, res)
                assert len(set(res)) == M and all(0 <= x < N for x in res)
                seen.add(tuple(res))
                cases += 1
            assert len(seen) == math.perm(N, M)
    assert cases == 10151


def test_algorithm1_unit_vectors():
    for line in _read_golden("algorithm1_units.txt"):
        head, r, res = [s.split() for s in line.split("|")]
        N, M = int(head[0]), int(head[1])
        assert [int(x) for x in oracle.algorithm1(M, N, [int(x) for x in r])] == [int(x) for x in res]


def test_algorithm1_rejects_bad_args():
    with pytest.raises(ValueError):
        oracle.algorithm1(5, 5, [0] * 5)      # M >= N is the caller's full-row case
    with pytest.raises(ValueError):
        oracle.algorithm1(2, 5, [0, 4])       # r_1 must be <= N-1-1 = 3


def test_algorithm1_large_random_vs_fisher_yates():
    rng = np.random.default_rng(7)
    for _ in range(2000):
        N = int(rng.integers(2, 5000))
        M = int(rng.integers(1, min(N, 64)))
        r = [int(rng.integers(0, N - i)) for i in range(M)]
        assert [int(x) for x in oracle.algorithm1(M, N, r)] == fisher_yates_partial(N, M, r)


def test_rng_contract_golden():
    for line in _read_golden("rng_contract.txt"):
        head, r, res = [s.split() for s in line.split("|")]
        seed, hop, node, N, M = int(head[0], 16), int(head[1]), int(head[2]), int(head[3]), int(head[4])
        got_r = [oracle.draw(seed, hop, node, i, N) for i in range(M)]
        assert got_r == [int(x) for x in r]
        adj = np.arange(N, dtype=np.int64) * 10   # positions recoverable from ids
        _, nbrs, pos = oracle.sample_hop([0, N], adj, [node], M, seed, hop)
        assert [int(x) for x in pos] == [int(x) for x in res]
        assert [int(x) for x in nbrs] == [10 * int(x) for x in res]


# ---------------------------------------------------------------- sampling op
def _same_row_many_nodes(N, K, base=1000):
    adj = np.arange(N, dtype=np.int64) + 10**6
    adj_ptr = np.arange(K + 1, dtype=np.int64) * N
    return adj_ptr, np.tile(adj, K), np.arange(base, base + K, dtype=np.int64)


def test_sample_marginals_uniform_chi2():
    """Each draw's position is uniform on [0, N) (a property of sampling without
    replacement): multinomial chi-square with N-1 dof per draw index, N=20, M=5,
    K=100,000 independent (node-keyed) rows."""
    N, M, K = 20, 5, 100_000
    adj_ptr, adj, T = _same_row_many_nodes(N, K)
    row_ptr, nbrs, pos = oracle.sample_hop(adj_ptr, adj, T, M, 0xABCDEF, 0)
    assert len(pos) == K * M
    P = pos.reshape(K, M)
    for i in range(M):
        c = np.bincount(P[:, i], minlength=N)
        assert stats.chisquare(c).pvalue > 1e-4, (i, c)
    # inclusion frequency of every position is M/N
    inc = np.bincount(pos, minlength=N)
    z = (inc - K * M / N) / math.sqrt(K * (M / N) * (1 - M / N))
    assert np.all(np.abs(z) < 5)
    assert np.all(np.sort(P, axis=1)[:, 1:] != np.sort(P, axis=1)[:, :-1])   # no repeats


def test_sample_ordered_pairs_uniform_chi2():
    """N=4, M=2: all 12 ordered pairs equally likely (chi-square, 11 dof)."""
    N, M, K = 4, 2, 60_000
    adj_ptr, adj, T = _same_row_many_nodes(N, K)
    _, _, pos = oracle.sample_hop(adj_ptr, adj, T, M, 0x7777, 1)
    P = pos.reshape(K, M)
    code = P[:, 0] * N + P[:, 1]
    c = np.bincount(code, minlength=N * N)
    valid = [a * N + b for a in range(N) for b in range(N) if a != b]
    assert c.sum() == c[valid].sum()
    assert stats.chisquare(c[valid]).pvalue > 1e-4


def test_sample_special_cases():
    """M >= N -> the full row in CSR order (A5); N = 0 -> empty (A6)."""
    adj_ptr = np.array([0, 0, 1, 5, 10, 11, 41], dtype=np.int64)
    adj = np.arange(41, dtype=np.int64) * 3 + 1
    T = np.array([7, 8, 9, 10, 11, 12], dtype=np.int64)
    row_ptr, nbrs, pos = oracle.sample_hop(adj_ptr, adj, T, 5, 99, 0)
    assert list(np.diff(row_ptr)) == [0, 1, 4, 5, 1, 5]
    assert list(nbrs[0:1]) == [adj[0]]
    assert list(nbrs[1:5]) == list(adj[1:5])
    assert list(nbrs[5:10]) == list(adj[5:10])           # N == M
    assert list(nbrs[10:11]) == list(adj[10:11])
    last = pos[11:16]
    assert len(set(last)) == 5 and all(0 <= p < 30 for p in last)
    assert list(nbrs[11:16]) == list(adj[11 + last])


def test_sample_determinism_and_keying():
    """Draws depend on (rng_seed, hop, node) only: same node at two positions of T
    gets the same sample; another hop or seed changes it."""
    N = 50
    adj_ptr = np.array([0, N, 2 * N, 3 * N], dtype=np.int64)
    adj = np.tile(np.arange(N, dtype=np.int64), 3)
    T = np.array([5, 6, 5], dtype=np.int64)
    _, nb, _ = oracle.sample_hop(adj_ptr, adj, T, 10, 1234, 0)
    assert list(nb[0:10]) == list(nb[20:30]) and list(nb[0:10]) != list(nb[10:20])
    _, nb2, _ = oracle.sample_hop(adj_ptr, adj, T, 10, 1234, 1)
    _, nb3, _ = oracle.sample_hop(adj_ptr, adj, T, 10, 1235, 0)
    assert list(nb2[0:10]) != list(nb[0:10]) and list(nb3[0:10]) != list(nb[0:10])


# ---------------------------------------------------------------- append unique
def check_append_unique(T, nbrs, U, sub_col, dup):
    """The invariants that determine first-appearance Append Unique uniquely
    (PAPER.md L160-166 + reading A7)."""
    nT = len(T)
    assert list(U[:nT]) == list(T)                              # targets first, in order
    assert len(set(U.tolist())) == len(U)                       # no duplicates
    assert set(U.tolist()) == set(T.tolist()) | set(nbrs.tolist())
    assert np.all(U[sub_col] == nbrs)                           # ids map back to the samples
    nxt = nT
    for p in range(len(nbrs)):                                  # new ids appear as nT, nT+1, ...
        if sub_col[p] >= nT:
            assert sub_col[p] <= nxt
            if sub_col[p] == nxt:
                nxt += 1
    assert nxt == len(U)
    assert np.array_equal(dup, np.bincount(sub_col, minlength=len(U)))


def test_append_unique_invariants_random():
    rng = np.random.default_rng(3)
    for trial in range(200):
        pool = int(rng.integers(1, 400))
        nT = int(rng.integers(0, min(pool, 60) + 1))
        T = rng.choice(pool, size=nT, replace=False).astype(np.int64)
        nbrs = rng.integers(0, pool, size=int(rng.integers(0, 500))).astype(np.int64)
        U, sub_col, dup = oracle.append_unique(T, nbrs)
        check_append_unique(T, nbrs, U, sub_col, dup)


def test_append_unique_worked_cases():
    # targets T0..T3 with ids 40,10,30,20 (the shape of PAPER.md Fig. 5, whose values are lost)
    T = np.array([40, 10, 30, 20], dtype=np.int64)
    nbrs = np.array([7, 10, 7, 50, 40, 8, 50], dtype=np.int64)
    U, sub_col, dup = oracle.append_unique(T, nbrs)
    assert list(U) == [40, 10, 30, 20, 7, 50, 8]
    assert list(sub_col) == [4, 1, 4, 5, 0, 6, 5]
    assert list(dup) == [1, 1, 0, 0, 2, 2, 1]
    # all neighbours are targets -> no new nodes (SURVEY 8(c) edge case)
    U, sub_col, _ = oracle.append_unique(T, np.array([20, 40, 40], dtype=np.int64))
    assert list(U) == [40, 10, 30, 20] and list(sub_col) == [3, 0, 0]
    # empty inputs
    U, sub_col, _ = oracle.append_unique(np.zeros(0, np.int64), np.zeros(0, np.int64))
    assert len(U) == 0 and len(sub_col) == 0


def test_append_unique_duplicate_target_is_error():
    with pytest.raises(oracle.DuplicateTargetError):
        oracle.append_unique(np.array([1, 2, 1], dtype=np.int64), np.array([3], dtype=np.int64))


# ---------------------------------------------------------------- gather
def test_gather_closed_form():
    """orc_gather rows == the generator's closed-form feature bytes, in input
    order, with repeats, from a shuffled table."""
    rng = np.random.default_rng(5)
    for dtype, dim in [("fp32", 32), ("fp16", 768), ("fp32", 3), ("fp16", 1)]:
        nodes = rng.permutation(1000).astype(np.int64)
        table = features.feature_bytes(42, nodes, dim, dtype)
        ids = rng.integers(0, 1000, size=777).astype(np.int64)
        X = oracle.gather(table, nodes, ids)
        assert np.array_equal(X, features.feature_bytes(42, ids, dim, dtype))
    assert oracle.gather(table, nodes, np.zeros(0, np.int64)).shape == (0, table.shape[1])


# ---------------------------------------------------------------- whole path
def test_minibatch_tiny_invariants():
    """Config-1 graph: every invariant of SURVEY.md 8(c) on the composed path."""
    p = presets.get("tiny")
    spec = p.graph()
    row_ptr, col = graph.csr(spec)

    def row_provider(T):
        starts, ends = row_ptr[T], row_ptr[T + 1]
        lens = ends - starts
        ptr = np.concatenate(([0], np.cumsum(lens)))
        idx = np.repeat(starts - ptr[:-1], lens) + np.arange(ptr[-1])
        return ptr, col[idx]

    def feat_provider(ids):
        u = np.unique(ids)
        return u, features.feature_bytes(presets.FEAT_SEED, u, p.feat_dim, p.feat_dtype)

    from synth import seeds as sd
    S = sd.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 0)
    out = oracle.minibatch(row_provider, feat_provider, S, p.fanouts, sd.rng_seed(presets.RNG_BASE, 0))
    prevU = S
    for h, hop in enumerate(out["hops"]):
        T = hop["targets"]
        assert np.array_equal(T, prevU)
        deg = row_ptr[T + 1] - row_ptr[T]
        assert np.array_equal(np.diff(hop["row_ptr"]), np.minimum(deg, p.fanouts[h]))
        for k in range(len(T)):
            a, b = hop["row_ptr"][k], hop["row_ptr"][k + 1]
            adjk = col[row_ptr[T[k]]:row_ptr[T[k] + 1]]
            assert len(set(hop["pos"][a:b].tolist())) == b - a
            assert np.array_equal(adjk[hop["pos"][a:b]], hop["nbrs"][a:b])
        check_append_unique(T, hop["nbrs"], hop["unique"], hop["sub_col"], hop["dup"])
        prevU = hop["unique"]
    assert np.array_equal(out["X"], features.feature_bytes(presets.FEAT_SEED, prevU, p.feat_dim, p.feat_dtype))


# ---------------------------------------------------------------- g-SpMM (NEXT #2)
def test_spmm_mean_pins():
    """orc_spmm_mean_*: mean of constant rows is the constant, empty rows give 0,
    linearity, and the adjoint identity <dy, A x> = <A^T dy, x> ties backward to forward."""
    rng = np.random.default_rng(2)
    nx, d = 50, 8
    deg = rng.integers(0, 6, size=30)
    rp = np.concatenate(([0], np.cumsum(deg)))
    col = rng.integers(0, nx, size=rp[-1]).astype(np.int32)
    x = np.ones((nx, d)) * 3.5
    y = oracle.spmm_mean_forward(rp, col, x)
    assert np.allclose(y[deg > 0], 3.5) and np.all(y[deg == 0] == 0)
    x1, x2 = rng.standard_normal((nx, d)), rng.standard_normal((nx, d))
    assert np.allclose(oracle.spmm_mean_forward(rp, col, 2 * x1 - x2),
                       2 * oracle.spmm_mean_forward(rp, col, x1) - oracle.spmm_mean_forward(rp, col, x2))
    dy = rng.standard_normal((30, d))
    lhs = np.sum(dy * oracle.spmm_mean_forward(rp, col, x1))
    rhs = np.sum(oracle.spmm_mean_backward(rp, col, dy, nx) * x1)
    assert abs(lhs - rhs) < 1e-9 * max(1, abs(lhs))
    # one row, explicit: mean of rows 1 and 3
    y = oracle.spmm_mean_forward([0, 2], np.array([1, 3], np.int32), x1)
    assert np.allclose(y[0], (x1[1] + x1[3]) / 2)
