"""Row-local power-law CSR generator (fixture; SURVEY.md section 8(d) "Generator formulas").

Shape targets: ogbn-products (2.45M nodes, ~124M CSR entries), ogbn-papers100M
(111M nodes, ~3.2B CSR entries, "8 bytes to store each edge")
and MAG240M (244M nodes, ~3.4B entries), plus a 10k-node tiny graph.

The adjacency list of node v is a pure function of (graph_seed, v):

  raw degree  d(v)   = min(d_max, floor(d_min / x^(3/4))),  x = 1 - u(gs, 0, v)
                        (a discrete Pareto tail with index beta = 4/3; x^(3/4) is
                        computed as sqrt(x) * sqrt(sqrt(x)) so that every step is a
                        correctly rounded IEEE op and the CUDA generator reproduces
                        it bit for bit)
  slot j      w(v,j) = min(n-1, floor(n * u^2 * sqrt(u))),  u = u(gs, 1, v, j)
                        (gamma = 2.5: low ids are in-degree hubs)
  row(v)             = sorted(set(w(v, j) for j < d(v)) - {v})

so the final degree is <= d(v).  Rows are sorted ascending, duplicate- and
self-loop-free.  Because rows are independent the oracle
can regenerate exactly the rows a batch touches, for any n.
"""

from dataclasses import dataclass

import numpy as np

from .hashing import h, unit

D_MAX_CAP = 1 << 17


@dataclass(frozen=True)
class GraphSpec:
    n: int                  # number of nodes
    d_min: float            # Pareto scale (calibrated so the CSR lands near the target E)
    graph_seed: int
    d_max: int = -1         # -1: min(n-1, 2^17)

    @property
    def dmax(self) -> int:
        return self.d_max if self.d_max >= 0 else min(self.n - 1, D_MAX_CAP)


def raw_degree(spec: GraphSpec, v) -> np.ndarray:
    v = np.asarray(v, dtype=np.int64)
    x = 1.0 - unit(h(spec.graph_seed, 0, v.astype(np.uint64)))
    t = np.sqrt(x)
    p = t * np.sqrt(t)
    val = np.floor(np.float64(spec.d_min) / p)
    val = np.minimum(val, np.float64(spec.dmax))
    return val.astype(np.int64)


def slot_dest(spec: GraphSpec, v, j) -> np.ndarray:
    u = unit(h(spec.graph_seed, 1, np.asarray(v, dtype=np.uint64), np.asarray(j, dtype=np.uint64)))
    c = (u * u) * np.sqrt(u)
    w = np.floor(np.float64(spec.n) * c).astype(np.int64)
    return np.minimum(w, spec.n - 1)


def rows(spec: GraphSpec, v, max_chunk: int = 1 << 24):
    """Final adjacency rows of the nodes in ``v`` (any order, repeats allowed).

    Returns (ptr int64[len(v)+1], col int64[ptr[-1]]): row k = col[ptr[k]:ptr[k+1]].
    """
    v = np.asarray(v, dtype=np.int64).reshape(-1)
    d = raw_degree(spec, v)
    ptr = np.zeros(len(v) + 1, dtype=np.int64)
    cols = []
    counts = np.zeros(len(v), dtype=np.int64)
    # chunk rows so that at most ~max_chunk raw slots are live at once
    csum = np.cumsum(d)
    lo = 0
    while lo < len(v):
        base = csum[lo - 1] if lo > 0 else 0
        hi = int(np.searchsorted(csum, base + max_chunk, side="right"))
        hi = max(hi, lo + 1)
        hi = min(hi, len(v))
        dv = d[lo:hi]
        tot = int(dv.sum())
        if tot:
            rid = np.repeat(np.arange(hi - lo, dtype=np.int64), dv)
            starts = np.concatenate(([0], np.cumsum(dv)[:-1]))
            j = np.arange(tot, dtype=np.int64) - np.repeat(starts, dv)
            vv = v[lo:hi][rid]
            w = slot_dest(spec, vv, j)
            key = rid * np.int64(spec.n) + w
            key = np.unique(key)                       # sorts, drops duplicates
            rid = key // spec.n
            w = key - rid * spec.n
            keep = w != v[lo:hi][rid]                  # drop self-loops
            rid, w = rid[keep], w[keep]
            counts[lo:hi] = np.bincount(rid, minlength=hi - lo)
            cols.append(w)
        lo = hi
    ptr[1:] = np.cumsum(counts)
    col = np.concatenate(cols) if cols else np.zeros(0, dtype=np.int64)
    return ptr, col


def csr(spec: GraphSpec):
    """Whole-graph CSR (row_ptr int64[n+1], col int64[E]) -- host, for small n."""
    return rows(spec, np.arange(spec.n, dtype=np.int64))


def shard_rows(n: int, rank: int, world: int) -> np.ndarray:
    """Global ids owned by ``rank`` under o(v) = v mod W, in local-row order l(v) = v div W
    (PAPER.md L110 hash partition)."""
    return np.arange(rank, n, world, dtype=np.int64)


# ------------------------------------------------------------------ native host generator
_native = None


def _native_lib():
    """synth/csrc/gen_host.cpp -> synth/libwggen_host.so (built on demand with g++)."""
    global _native
    if _native is None:
        import ctypes
        import os
        import subprocess
        here = os.path.dirname(os.path.abspath(__file__))
        src = os.path.join(here, "csrc", "gen_host.cpp")
        so = os.path.join(here, "libwggen_host.so")
        if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
            tmp = so + f".tmp{os.getpid()}"
            subprocess.check_call(["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-shared", "-fPIC", src, "-o", tmp])
            os.replace(tmp, so)
        L = ctypes.CDLL(so)
        P = ctypes.c_void_p
        L.genh_rows.argtypes = [ctypes.c_int64, ctypes.c_double, ctypes.c_int64, ctypes.c_uint64, P, ctypes.c_int64,
                                P, P]
        L.genh_rows.restype = ctypes.c_int
        L.genh_features.argtypes = [ctypes.c_uint64, P, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, P]
        L.genh_features.restype = ctypes.c_int
        _native = L
    return _native


def rows_native(spec: GraphSpec, v):
    """Same result as rows(), computed by the C++ host generator (fast)."""
    import ctypes
    L = _native_lib()
    v = np.ascontiguousarray(np.asarray(v, dtype=np.int64).reshape(-1))
    ptr = np.zeros(len(v) + 1, dtype=np.int64)
    vp = v.ctypes.data_as(ctypes.c_void_p) if len(v) else None
    L.genh_rows(spec.n, float(spec.d_min), spec.dmax, spec.graph_seed, vp, len(v),
                ptr.ctypes.data_as(ctypes.c_void_p), None)
    col = np.zeros(max(int(ptr[-1]), 1), dtype=np.int64)
    L.genh_rows(spec.n, float(spec.d_min), spec.dmax, spec.graph_seed, vp, len(v),
                ptr.ctypes.data_as(ctypes.c_void_p), col.ctypes.data_as(ctypes.c_void_p))
    return ptr, col[: ptr[-1]]
