"""Procedural node features (fixture; SURVEY.md 8(d) "Feature values").

bits(v, c) derive from hv = h(feat_seed, v, c):
  fp32: 0x3F800000 | (hv >> 41)     -> values in [1, 2)
  fp16: 0x3C00     | (hv >> 54)     -> values in [1, 2)
  bf16: 0x3F80     | (hv >> 57)     -> values in [1, 2)
All finite; parity compares the integer views (the gather is a byte copy,
PAPER.md L176).
"""

import numpy as np

from .hashing import h

DTYPES = {"fp32": (4, np.uint32), "fp16": (2, np.uint16), "bf16": (2, np.uint16)}
WG_DTYPE_CODE = {"fp32": 0, "fp16": 1, "bf16": 2}


def elt_bytes(dtype: str) -> int:
    return DTYPES[dtype][0]


def feature_bits(feat_seed: int, v, dim: int, dtype: str) -> np.ndarray:
    """Integer view [len(v), dim] of the feature rows of nodes v."""
    v = np.asarray(v, dtype=np.int64).reshape(-1, 1).astype(np.uint64)
    c = np.arange(dim, dtype=np.uint64).reshape(1, -1)
    hv = h(feat_seed, v, c)
    if dtype == "fp32":
        return (np.uint64(0x3F800000) | (hv >> np.uint64(41))).astype(np.uint32)
    if dtype == "fp16":
        return (np.uint64(0x3C00) | (hv >> np.uint64(54))).astype(np.uint16)
    if dtype == "bf16":
        return (np.uint64(0x3F80) | (hv >> np.uint64(57))).astype(np.uint16)
    raise ValueError(dtype)


def feature_bytes(feat_seed: int, v, dim: int, dtype: str) -> np.ndarray:
    """Row bytes [len(v), dim*elt] (uint8) of nodes v."""
    b = feature_bits(feat_seed, v, dim, dtype)
    return b.view(np.uint8).reshape(b.shape[0], dim * DTYPES[dtype][0])


def feature_bytes_native(feat_seed: int, v, dim: int, dtype: str) -> np.ndarray:
    """Same bytes as feature_bytes(), computed by the C++ host generator (fast)."""
    import ctypes
    from .graph import _native_lib
    v = np.ascontiguousarray(np.asarray(v, dtype=np.int64).reshape(-1))
    eb, _ = DTYPES[dtype]
    out = np.zeros((len(v), dim * eb), dtype=np.uint8)
    if len(v) and dim:
        _native_lib().genh_features(feat_seed, v.ctypes.data_as(ctypes.c_void_p), len(v), dim,
                                    WG_DTYPE_CODE[dtype], out.ctypes.data_as(ctypes.c_void_p))
    return out
