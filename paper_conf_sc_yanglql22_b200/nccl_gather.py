"""The distributed-memory global gather the paper compares against (PAPER.md L178-180,
Fig. 4 left; Fig. 10: "P2P gather ... at least 2x faster"):

    1 bucket the ids by home GPU          (wg_bucket_by_owner, CUDA)
    2 all-to-all the counts, then the ids (torch.distributed: NCCL, or gloo via host)
    3 local gather of the received ids    (wg_gather; every received id is owned here)
    4 all-to-all the feature rows back
    5 reorder into input order            (wg_rows_permute, CUDA)

It is the baseline, not the product: the product is DSM.gather, one kernel of P2P loads.
"""

import ctypes

import torch
import torch.distributed as dist

from ._lib import check, lib


def _p(t):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else None


class DistributedGather:
    def __init__(self, dsm, group=None):
        self.dsm = dsm
        self.group = group
        self.world = dsm.world
        self.host_comm = dist.get_backend(group) != "nccl" if self.world > 1 else False

    def _a2a(self, out, inp, out_splits, in_splits):
        if self.world == 1:
            out.copy_(inp)
            return
        if self.host_comm:  # gloo: exchange through host memory
            o = torch.empty(out.shape, dtype=out.dtype)
            dist.all_to_all_single(o, inp.cpu(), out_splits, in_splits, group=self.group)
            out.copy_(o)
        else:
            dist.all_to_all_single(out, inp, out_splits, in_splits, group=self.group)

    def gather(self, ids, out=None):
        d = self.dsm
        dev = d.device
        n = ids.numel()
        st = ctypes.c_void_p(torch.cuda.current_stream(dev).cuda_stream)
        counts = torch.zeros(2 * self.world, dtype=torch.int64, device=dev)
        bucketed = torch.empty(max(n, 1), dtype=torch.int64, device=dev)
        perm = torch.empty(max(n, 1), dtype=torch.int64, device=dev)
        check(lib().wg_bucket_by_owner(d.h, _p(ids), n, None, _p(counts), _p(bucketed), _p(perm), st))   # step 1
        send_counts = counts[: self.world]
        recv_counts = torch.empty_like(send_counts)
        self._a2a(recv_counts, send_counts, None, None)                                                   # step 2a
        sc, rc = send_counts.tolist(), recv_counts.tolist()
        req = torch.empty(max(sum(rc), 1), dtype=torch.int64, device=dev)
        self._a2a(req[: sum(rc)], bucketed[:n], rc, sc)                                                   # step 2b
        rb = d.row_bytes
        local = torch.empty((max(sum(rc), 1), rb), dtype=torch.uint8, device=dev)
        if sum(rc):
            check(lib().wg_gather(d.h, _p(req), sum(rc), None, _p(local), st))                            # step 3
        back = torch.empty((max(n, 1), rb), dtype=torch.uint8, device=dev)
        self._a2a(back[:n].view(-1), local[: sum(rc)].view(-1), [c * rb for c in sc], [c * rb for c in rc])  # 4
        if out is None:
            out = torch.empty((max(n, 1), rb), dtype=torch.uint8, device=dev)
        check(lib().wg_rows_permute(_p(back), _p(out), _p(perm), n, rb, st))                              # step 5
        return out
