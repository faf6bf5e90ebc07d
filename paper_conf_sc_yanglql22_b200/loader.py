"""Setup helpers: build a DSM for one of the synthetic presets (not on the hot path).

Small graphs are generated on the host (synth.graph) and copied in; large ones are
generated per shard directly on the device (synth.gpu).  Either way the rows are
identical (tests/test_gpu_synth.py).
"""

import time

import numpy as np
import torch

from synth import features as sfeat
from synth import graph as sgraph
from synth import presets as spre

from .dsm import DSM, local_num_edges
from .pipeline import required_keys


def build_dsm(preset, rank=0, world=1, device=None, allgather=None, max_seeds=None, on_device=None,
              feat_dim=None, feat_dtype=None, extra_keys=0, flags=0, col32=None):
    """Create and fill a DSM for ``preset`` (a synth.presets.Preset).  Returns (dsm, info).
    ``flags``: wg_dsm_desc.flags (e.g. WG_DSM_CSR_REPLICATED: every rank holds the whole CSR).
    ``col32``: store col_idx as uint32 (WG_DSM_COL32); default: whenever the node ids fit (n < 2^31)."""
    from ._lib import WG_DSM_COL32, WG_DSM_CSR_REPLICATED
    if col32 is None:
        col32 = preset.n < (1 << 31)
    if col32:
        flags |= WG_DSM_COL32
    csr_rep = bool(flags & WG_DSM_CSR_REPLICATED)
    c_rank, c_world = (0, 1) if csr_rep else (rank, world)   # which CSR rows this rank's slab holds
    device = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    spec = preset.graph()
    fd = preset.feat_dim if feat_dim is None else feat_dim
    fdt = preset.feat_dtype if feat_dtype is None else feat_dtype
    S = preset.seeds_per_batch if max_seeds is None else max_seeds
    keys = max(required_keys(spec.n, preset.fanouts, S), extra_keys, 1)
    on_device = (spec.n > 200_000) if on_device is None else on_device
    info = {}
    t0 = time.perf_counter()
    if on_device:
        from synth import gpu as sgpu
        rp, col = sgpu.shard_csr_gpu(spec, c_rank, c_world, device)
        e_local = col.numel()
    else:
        g_rp, g_col = sgraph.csr(spec)
        e_local = local_num_edges(g_rp, c_rank, c_world)
    info["gen_s"] = time.perf_counter() - t0
    if on_device:
        torch.cuda.empty_cache()  # return the generator's temporaries to the driver before the big slab
    t1 = time.perf_counter()
    dsm = DSM(spec.n, e_local, fd, fdt, keys, rank=rank, world_size=world, device=device.index, allgather=allgather,
              flags=flags)
    torch.cuda.synchronize(device)
    info["create_s"] = time.perf_counter() - t1
    if on_device:
        lrp, lcol, lfeat = dsm.local_view()
        lrp.copy_(rp)
        if e_local:
            lcol.copy_(col)
        del rp, col
        if fd:
            from synth import gpu as sgpu
            sgpu.fill_dsm_features_gpu(dsm, spre.FEAT_SEED, rank, world, fd, sfeat.WG_DTYPE_CODE[fdt])
    else:
        dsm.fill_from_global_csr(g_rp, g_col)
        if fd:
            v = sgraph.shard_rows(spec.n, rank, world)
            dsm.fill_features(sfeat.feature_bytes(spre.FEAT_SEED, v, fd, fdt))
    torch.cuda.synchronize(device)
    if allgather is not None and world > 1:
        allgather(None, None, 0, None)  # barrier: every shard filled before anyone reads
    info["e_local"] = e_local
    info["fill_s"] = time.perf_counter() - t0 - info["gen_s"] - info["create_s"]
    return dsm, info
