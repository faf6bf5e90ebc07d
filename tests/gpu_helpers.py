"""Shared helpers for the -m gpu parity tests: run the CUDA path through the C ABI
(python binding) and the CPU oracle on the same seeded inputs."""

import numpy as np
import torch

import oracle
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import providers


def csr_from_rows(rows):
    rp = np.zeros(len(rows) + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    col = np.concatenate([np.asarray(r, dtype=np.int64) for r in rows]) if rp[-1] else np.zeros(0, np.int64)
    return rp, col


def make_dsm(row_ptr, col, feat_rows=None, feat_dim=0, feat_dtype="fp32", max_keys=1 << 16, rank=0, world=1,
             allgather=None, flags=0):
    n = len(row_ptr) - 1
    e_local = len(col) if flags & pkg.WG_DSM_CSR_REPLICATED else pkg.local_num_edges(row_ptr, rank, world)
    dsm = pkg.DSM(n, e_local, feat_dim, feat_dtype, max_keys, rank=rank,
                  world_size=world, allgather=allgather, flags=flags)
    dsm.fill_from_global_csr(row_ptr, col)
    if feat_dim:
        dsm.fill_features(feat_rows[rank::world])
    torch.cuda.synchronize()
    if allgather is not None and world > 1:
        allgather(None, None, 0, None)
    return dsm


def oracle_hop(row_ptr, col, T, M, seed, hop):
    rows = providers.host_row_provider(None, row_ptr, col)
    adj_ptr, adj = rows(np.asarray(T, dtype=np.int64))
    return oracle.sample_hop(adj_ptr, adj, T, M, seed, hop)


def gpu_hop(dsm, T, M, seed, hop):
    t = torch.from_numpy(np.asarray(T, dtype=np.int64)).cuda()
    rp, nb, pos, ne = dsm.sample_neighbors(t, M, seed, hop, with_pos=True)
    torch.cuda.synchronize()
    e = int(ne.item())
    return rp.cpu().numpy(), nb[:e].cpu().numpy(), pos[:e].cpu().numpy()


def gpu_unique(dsm, T, nbrs, with_dup=True):
    t = torch.from_numpy(np.asarray(T, dtype=np.int64)).cuda()
    nb = torch.from_numpy(np.asarray(nbrs, dtype=np.int64)).cuda()
    U, nU, sc, dup = dsm.append_unique(t, nb, with_dup=with_dup)
    torch.cuda.synchronize()
    u = int(nU.item())
    return U[:u].cpu().numpy(), sc[:len(nbrs)].cpu().numpy(), (dup[:u].cpu().numpy() if with_dup else None)


def gpu_sample_hop(dsm, T, M, seed, hop):
    """One fused hop (wg_sample_hop, no side stream): row_ptr, nbrs, pos, U, sub_col, dup."""
    t = torch.from_numpy(np.asarray(T, dtype=np.int64)).cuda()
    o = dsm.sample_hop(t, M, seed, hop, with_pos=True, with_dup=True)
    torch.cuda.synchronize()
    e, u = int(o["num_edges"].item()), int(o["num_unique"].item())
    return (o["row_ptr"].cpu().numpy(), o["nbrs"][:e].cpu().numpy(), o["pos"][:e].cpu().numpy(),
            o["unique"][:u].cpu().numpy(), o["sub_col"][:e].cpu().numpy(), o["dup"][:u].cpu().numpy())


def oracle_sample_hop(row_ptr, col, T, M, seed, hop):
    """The fused hop's definition: oracle sampling, then oracle append-unique of its neighbours."""
    rp, nb, pos = oracle_hop(row_ptr, col, T, M, seed, hop)
    U, sc, dup = oracle.append_unique(np.asarray(T, dtype=np.int64), nb)
    return rp, nb, pos, U, sc, dup
