"""splitmix64 and the word-folding hash h(w0, w1, ...) used by every generator.

h(w0)          = splitmix64(w0)
h(w0, ..., wk) = splitmix64(h(w0, ..., w_{k-1}) ^ wk)
u(...)         = (h(...) >> 11) * 2**-53          in [0, 1)

The same definitions are implemented for the GPU generator in
``synth/csrc/gen.cu``; ``tests/test_synth.py`` checks that the two agree.
"""

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_S30, _S27, _S31, _S11 = np.uint64(30), np.uint64(27), np.uint64(31), np.uint64(11)


def splitmix64(x):
    """splitmix64 finaliser (Steele, Lea, Flood 2014) on a uint64 array (wrapping)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + _GOLDEN
        z = (z ^ (z >> _S30)) * _M1
        z = (z ^ (z >> _S27)) * _M2
    return z ^ (z >> _S31)


def splitmix64_int(x: int) -> int:
    """Scalar Python-int version (for per-batch seeds)."""
    m = (1 << 64) - 1
    z = (x + 0x9E3779B97F4A7C15) & m
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & m
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & m
    return z ^ (z >> 31)


def h(*words):
    """Fold splitmix64 over the words (each a scalar or a broadcastable array)."""
    s = splitmix64(np.asarray(words[0], dtype=np.uint64))
    for w in words[1:]:
        s = splitmix64(s ^ np.asarray(w, dtype=np.uint64))
    return s


def unit(hv):
    """(h >> 11) * 2^-53: exact float64 in [0, 1)."""
    return (np.asarray(hv, dtype=np.uint64) >> _S11).astype(np.float64) * (2.0 ** -53)
