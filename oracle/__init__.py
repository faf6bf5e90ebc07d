"""CPU oracle of WholeGraph's mini-batch preparation path -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  It
shares no code with the CUDA path (``paper_conf_sc_yanglql22_b200``); the only
thing both sides import is the seeded input generator package ``synth``.

The arithmetic lives in ``oracle/oracle.cpp`` (plain single-threaded C++17,
``g++ -O2``); this module compiles it on demand and marshals numpy arrays.
Each function cites the PAPER.md passage it follows; see oracle.cpp for the
per-function pin status.
"""

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.cpp -> liboracle.so (single-threaded, -O2, no OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        L.orc_philox4x32_10.argtypes = [P, P, P]
        L.orc_philox4x32_10.restype = None
        L.orc_draw.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_uint32]
        L.orc_draw.restype = ctypes.c_uint32
        L.orc_algorithm1.argtypes = [ctypes.c_int32, ctypes.c_uint32, P, P]
        L.orc_algorithm1.restype = ctypes.c_int
        L.orc_sample_hop.argtypes = [P, P, P, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64,
                                     ctypes.c_int32, P, P, P]
        L.orc_sample_hop.restype = ctypes.c_int64
        L.orc_append_unique.argtypes = [P, ctypes.c_int64, P, ctypes.c_int64, P, P, P, P]
        L.orc_append_unique.restype = ctypes.c_int
        L.orc_gather.argtypes = [P, P, ctypes.c_int64, ctypes.c_int64, P, ctypes.c_int64, P]
        L.orc_gather.restype = ctypes.c_int
        L.orc_spmm_mean_forward.argtypes = [P, ctypes.c_int64, P, P, ctypes.c_int64, P]
        L.orc_spmm_mean_forward.restype = None
        L.orc_spmm_mean_backward.argtypes = [P, ctypes.c_int64, P, P, ctypes.c_int64, P, ctypes.c_int64]
        L.orc_spmm_mean_backward.restype = None
        _lib = L
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def philox4x32_10(ctr, key):
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    lib().orc_philox4x32_10(_p(c), _p(k), _p(out))
    return out


def draw(rng_seed: int, hop: int, node: int, i: int, N: int) -> int:
    """r_i of Algorithm 1 line 1 under reading A3."""
    return int(lib().orc_draw(rng_seed, hop, node, i, N))


def algorithm1(M: int, N: int, r):
    """Algorithm 1 on given draws r[0..M-1]; returns res[M]."""
    r = np.ascontiguousarray(r, dtype=np.uint32)
    res = np.zeros(M, dtype=np.uint32)
    rc = lib().orc_algorithm1(M, N, _p(r), _p(res))
    if rc != 0:
        raise ValueError("algorithm1: bad arguments")
    return res


def sample_hop(adj_ptr, adj, T, M: int, rng_seed: int, hop: int):
    """One sampling hop.  Row k of (adj_ptr, adj) is T[k]'s adjacency.
    Returns (out_row_ptr int64[nT+1], nbrs int64[E], pos int32[E])."""
    adj_ptr = np.ascontiguousarray(adj_ptr, dtype=np.int64)
    adj = np.ascontiguousarray(adj, dtype=np.int64)
    T = np.ascontiguousarray(T, dtype=np.int64)
    deg = np.diff(adj_ptr)
    cap = int(np.minimum(deg, M).sum())
    out_row_ptr = np.zeros(len(T) + 1, dtype=np.int64)
    nbrs = np.zeros(max(cap, 1), dtype=np.int64)
    pos = np.zeros(max(cap, 1), dtype=np.int32)
    e = lib().orc_sample_hop(_p(adj_ptr), _p(adj if len(adj) else np.zeros(1, np.int64)), _p(T), len(T),
                             M, rng_seed, hop, _p(out_row_ptr), _p(nbrs), _p(pos))
    if e < 0:
        raise ValueError("sample_hop: bad arguments")
    return out_row_ptr, nbrs[:e], pos[:e]


class DuplicateTargetError(ValueError):
    pass


def append_unique(T, nbrs):
    """Append Unique with first-appearance numbering (A7).
    Returns (U int64[nU], sub_col int32[E], dup int32[nU])."""
    T = np.ascontiguousarray(T, dtype=np.int64)
    nbrs = np.ascontiguousarray(nbrs, dtype=np.int64)
    cap = len(T) + len(nbrs)
    U = np.zeros(max(cap, 1), dtype=np.int64)
    nU = np.zeros(1, dtype=np.int64)
    sub_col = np.zeros(max(len(nbrs), 1), dtype=np.int32)
    dup = np.zeros(max(cap, 1), dtype=np.int32)
    rc = lib().orc_append_unique(_p(T), len(T), _p(nbrs), len(nbrs), _p(U), _p(nU), _p(sub_col), _p(dup))
    if rc == 1:
        raise DuplicateTargetError("duplicate target")
    if rc != 0:
        raise ValueError("append_unique: bad arguments")
    u = int(nU[0])
    return U[:u], sub_col[:len(nbrs)], dup[:u]


def gather(table_rows, table_ids, ids):
    """Global gather: out[i] = row of node ids[i]; table_rows is
    uint8 [n_rows, row_bytes] holding nodes table_ids."""
    table_rows = np.ascontiguousarray(table_rows, dtype=np.uint8)
    table_ids = np.ascontiguousarray(table_ids, dtype=np.int64)
    ids = np.ascontiguousarray(ids, dtype=np.int64)
    rb = table_rows.shape[1]
    out = np.zeros((len(ids), rb), dtype=np.uint8)
    rc = lib().orc_gather(_p(table_rows), _p(table_ids), len(table_ids), rb, _p(ids), len(ids), _p(out))
    if rc != 0:
        raise ValueError("gather: id without a table row")
    return out


def spmm_mean_forward(row_ptr, col, x):
    """g-SpMM mean aggregation forward, float64."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    x = np.ascontiguousarray(x, dtype=np.float64)
    n = len(row_ptr) - 1
    y = np.zeros((n, x.shape[1]), dtype=np.float64)
    lib().orc_spmm_mean_forward(_p(row_ptr), n, _p(col if len(col) else np.zeros(1, np.int32)), _p(x), x.shape[1], _p(y))
    return y


def spmm_mean_backward(row_ptr, col, dy, n_x_rows):
    """g-SpMM mean aggregation backward (gradient w.r.t. x), float64."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    dy = np.ascontiguousarray(dy, dtype=np.float64)
    n = len(row_ptr) - 1
    dx = np.zeros((n_x_rows, dy.shape[1]), dtype=np.float64)
    lib().orc_spmm_mean_backward(_p(row_ptr), n, _p(col if len(col) else np.zeros(1, np.int32)), _p(dy), dy.shape[1],
                                 _p(dx), n_x_rows)
    return dx


def minibatch(row_provider, feat_provider, seeds, fanouts, rng_seed: int, timer=None):
    """The whole path (SURVEY.md 8(c) ORACLE): for each hop, sample then append
    unique, T_{h+1} = U_h (reading A10); finally gather U_{H-1}.

    row_provider(T) -> (adj_ptr, adj) and feat_provider(ids) -> (table_ids,
    uint8 rows) (a table holding at least those nodes, in any order) come from
    the input generators; ``timer`` (optional) is a context-manager factory
    wrapped around the oracle's own work only (used by bench.py's cpu_baseline).
    Returns a dict with per-hop arrays and the gathered bytes."""
    import contextlib
    timer = timer or contextlib.nullcontext
    T = np.asarray(seeds, dtype=np.int64)
    hops = []
    for h, M in enumerate(fanouts):
        adj_ptr, adj = row_provider(T)
        with timer():
            row_ptr, nbrs, pos = sample_hop(adj_ptr, adj, T, M, rng_seed, h)
            U, sub_col, dup = append_unique(T, nbrs)
        hops.append(dict(targets=T, row_ptr=row_ptr, nbrs=nbrs, pos=pos, unique=U, sub_col=sub_col, dup=dup))
        T = U
    table_ids, table = feat_provider(T)
    with timer():
        X = gather(table, table_ids, T)
    return dict(hops=hops, X=X)
