"""Host-side row / feature providers for the CPU oracle (test infrastructure, no method
arithmetic): adjacency rows of a list of nodes and their feature bytes, from a host CSR or
regenerated from the seeded generator.  Used by tests/, smoke() and bench.py's oracle legs."""

import numpy as np

from . import features as sfeat
from . import graph as sgraph
from . import presets as spre


def host_row_provider(spec, row_ptr=None, col=None):
    """Adjacency rows for the oracle: slices of a host CSR if given, else regenerated
    per node from the generator (any n)."""
    if row_ptr is not None:
        def rows(T):
            T = np.asarray(T, dtype=np.int64)
            starts, ends = row_ptr[T], row_ptr[T + 1]
            lens = ends - starts
            ptr = np.zeros(len(T) + 1, dtype=np.int64)
            ptr[1:] = np.cumsum(lens)
            idx = np.repeat(starts - ptr[:-1], lens) + np.arange(ptr[-1], dtype=np.int64)
            return ptr, col[idx]
        return rows
    return lambda T: sgraph.rows_native(spec, T)


def host_feat_provider(preset, feat_dim=None, feat_dtype=None):
    """Feature bytes of a set of nodes: (sorted unique ids, their rows)."""
    fd = preset.feat_dim if feat_dim is None else feat_dim
    fdt = preset.feat_dtype if feat_dtype is None else feat_dtype

    def feats(ids):
        u = np.unique(np.asarray(ids, dtype=np.int64))
        return u, sfeat.feature_bytes_native(spre.FEAT_SEED, u, fd, fdt)
    return feats
