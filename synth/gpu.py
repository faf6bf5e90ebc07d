"""Device-side fill of the synthetic inputs (same formulas as synth/graph.py and
synth/features.py; kernels in synth/csrc/gen.cu -> synth/libwggen.so).

Fixture code: it builds inputs, it does not run the method.  torch supplies the
temporaries and the prefix sums.
"""

import ctypes
import os
import subprocess

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "csrc", "gen.cu")
LIB = os.path.join(_HERE, "libwggen.so")
_lib = None


def build(force=False):
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(_SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-std=c++17", "-Xcompiler", "-fPIC", "-shared", "-cudart", "static", _SRC, "-o", tmp])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB):
            raise ImportError(f"{LIB} missing; run __graft_entry__.build()")
        L = ctypes.CDLL(LIB)
        P, I, I64, U64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_uint64
        L.gen_raw_degree.argtypes = [I64, I, I, ctypes.c_double, I64, U64, I64, P, P]
        L.gen_fill_raw.argtypes = [I64, I, I, U64, I64, P, P, P]
        L.gen_segmented_sort.argtypes = [P, ctypes.POINTER(ctypes.c_size_t), P, P, I, I, P, P]
        L.gen_dedup_count.argtypes = [I, I, I64, P, P, P, P]
        L.gen_compact.argtypes = [I, I, I64, P, P, P, P, P]
        L.gen_features.argtypes = [U64, I, I, I64, I64, I, I64, P, I64, I64, P, P]
        _lib = L
    return _lib


def _ck(rc):
    if rc != 0:
        raise RuntimeError(f"generator CUDA error {rc}")


def _p(t):
    return ctypes.c_void_p(t.data_ptr())


def n_local(n, rank, world):
    return (n - rank + world - 1) // world if n > rank else 0


def shard_csr_gpu(spec, rank, world, device, max_sort_items=1 << 30):
    """Rows v = rank, rank+W, ... of the generator graph (local row l = v div W),
    built on ``device``.  Returns (row_ptr int64[n_local+1], col int64[E_local])."""
    L = lib()
    st = ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)
    nl = n_local(spec.n, rank, world)
    i64 = dict(dtype=torch.int64, device=device)
    deg = torch.empty(max(nl, 1), **i64)
    _ck(L.gen_raw_degree(spec.n, rank, world, float(spec.d_min), spec.dmax, spec.graph_seed, nl, _p(deg), st))
    raw_off = torch.zeros(nl + 1, **i64)
    torch.cumsum(deg[:nl], 0, out=raw_off[1:])
    e_raw = int(raw_off[-1].item())
    raw = torch.empty(max(e_raw, 1), **i64)
    _ck(L.gen_fill_raw(spec.n, rank, world, spec.graph_seed, nl, _p(raw_off), _p(raw), st))
    srt = torch.empty_like(raw)
    # segmented sort in row chunks of < max_sort_items entries
    off_host = raw_off.cpu().numpy()
    lo = 0
    while lo < nl:
        hi = int(np.searchsorted(off_host, off_host[lo] + max_sort_items, side="right")) - 1
        hi = min(max(hi, lo + 1), nl)
        base = int(off_host[lo])
        items = int(off_host[hi] - base)
        if items > 0:
            rel = (raw_off[lo:hi + 1] - base).to(torch.int32)
            tb = ctypes.c_size_t(0)
            kin = raw[base:]
            kout = srt[base:]
            _ck(L.gen_segmented_sort(None, ctypes.byref(tb), _p(kin), _p(kout), items, hi - lo, _p(rel), st))
            tmp = torch.empty(max(tb.value, 1), dtype=torch.uint8, device=device)
            _ck(L.gen_segmented_sort(_p(tmp), ctypes.byref(tb), _p(kin), _p(kout), items, hi - lo, _p(rel), st))
            del tmp
        lo = hi
    del raw
    _ck(L.gen_dedup_count(rank, world, nl, _p(raw_off), _p(srt), _p(deg), st))
    row_ptr = torch.zeros(nl + 1, **i64)
    torch.cumsum(deg[:nl], 0, out=row_ptr[1:])
    e = int(row_ptr[-1].item())
    col = torch.empty(max(e, 1), **i64)
    _ck(L.gen_compact(rank, world, nl, _p(raw_off), _p(srt), _p(row_ptr), _p(col), st))
    torch.cuda.current_stream(device).synchronize()
    return row_ptr, col[:e]


def fill_features_gpu(feat_view_u8, feat_seed, rank, world, dim, dtype_code, tail_view_u8=None, body_bytes=0):
    """Write bits(v, c) into a shard view uint8 [n_local, stride]; with a tail view (the DSM's split
    row layout, DSM.tail_view()) bytes >= body_bytes of each row go to the tail view instead."""
    L = lib()
    dev = feat_view_u8.device
    st = ctypes.c_void_p(torch.cuda.current_stream(dev).cuda_stream)
    nl, stride = feat_view_u8.shape
    tp = tail_view_u8.stride(0) if tail_view_u8 is not None else 0
    _ck(L.gen_features(feat_seed, rank, world, nl, dim, dtype_code, stride, _p(feat_view_u8), body_bytes, tp,
                       _p(tail_view_u8) if tail_view_u8 is not None else None, st))


def fill_dsm_features_gpu(dsm, feat_seed, rank, world, dim, dtype_code):
    """fill_features_gpu into a DSM's shard, honouring its row layout."""
    _, _, fv = dsm.local_view()
    fill_features_gpu(fv, feat_seed, rank, world, dim, dtype_code, dsm.tail_view(), dsm.body_bytes)
