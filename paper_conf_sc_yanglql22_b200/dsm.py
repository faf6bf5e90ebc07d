"""Python side of the DSM and the three ops (marshalling only).

PyTorch is used for device memory, streams and process groups; every step of
the path runs in libwg.so's sm_100a kernels (include/wg.h).
"""

import ctypes
import threading

import numpy as np
import torch

from . import _lib
from ._lib import check, lib

DTYPE_CODE = {"fp32": 0, "fp16": 1, "bf16": 2}
DTYPE_TORCH = {"fp32": torch.float32, "fp16": torch.float16, "bf16": torch.bfloat16}
DTYPE_BYTES = {"fp32": 4, "fp16": 2, "bf16": 2}


def _ptr(t):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else None


def _stream(stream):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


class _CudaArray:
    """Zero-copy view of raw device memory through __cuda_array_interface__."""

    def __init__(self, ptr, shape, typestr):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (ptr, False),
                                         "version": 2, "strides": None}


def device_view(ptr: int, shape, dtype: torch.dtype, device) -> torch.Tensor:
    typestr = {torch.int64: "<i8", torch.uint8: "|u1", torch.int32: "<i4"}[dtype]
    if int(np.prod(shape)) == 0:
        return torch.empty(shape, dtype=dtype, device=device)
    return torch.as_tensor(_CudaArray(ptr, shape, typestr), device=device)


# ------------------------------------------------------------------ allgather callbacks
class TorchDistAllgather:
    """Allgather of host bytes over a torch.distributed process group (NCCL or gloo).
    Used only at DSM create/destroy, never on the hot path."""

    def __init__(self, group=None, device=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        backend = dist.get_backend(group)
        self.dev = device if backend == "nccl" else torch.device("cpu")
        self.world = dist.get_world_size(group)

    def __call__(self, send, recv, nbytes, ctx):
        try:
            n = max(int(nbytes), 1)
            src = torch.zeros(n, dtype=torch.uint8)
            if nbytes:
                ctypes.memmove(src.data_ptr(), send, nbytes)
            src = src.to(self.dev)
            outs = [torch.empty(n, dtype=torch.uint8, device=self.dev) for _ in range(self.world)]
            self.dist.all_gather(outs, src, group=self.group)
            if nbytes:
                out = torch.cat(outs).cpu().contiguous()
                ctypes.memmove(recv, out.data_ptr(), nbytes * self.world)
            return 0
        except Exception as e:  # pragma: no cover - surfaced as WG_ERR_COLLECTIVE
            print("allgather failed:", e)
            return 1


class ThreadAllgather:
    """Allgather among W threads of ONE process (in-process virtual ranks sharing a
    GPU): used to test the W > 1 addressing on a single device."""

    def __init__(self, world):
        self.world = world
        self.barrier = threading.Barrier(world)
        self.slots = [None] * world
        self.local = threading.local()

    def for_rank(self, rank):
        def fn(send, recv, nbytes, ctx):
            try:
                self.slots[rank] = ctypes.string_at(send, nbytes) if nbytes else b""
                self.barrier.wait()
                if nbytes:
                    blob = b"".join(self.slots)
                    ctypes.memmove(recv, blob, len(blob))
                self.barrier.wait()
                return 0
            except Exception as e:  # pragma: no cover
                print("thread allgather failed:", e)
                return 1
        return fn


# ------------------------------------------------------------------ DSM
class DSM:
    """The multi-GPU distributed shared memory holding one row-sharded CSR graph and
    its feature table.  Collective create/destroy."""

    def __init__(self, num_nodes, local_num_edges, feat_dim=0, feat_dtype="fp32", max_batch_keys=1 << 20,
                 rank=0, world_size=1, device=None, allgather=None, flags=0):
        if device is None:
            device = torch.cuda.current_device()
        self.device = torch.device("cuda", device) if isinstance(device, int) else torch.device(device)
        self.rank, self.world = rank, world_size
        self.num_nodes, self.feat_dim, self.feat_dtype = num_nodes, feat_dim, feat_dtype
        self.row_bytes = feat_dim * DTYPE_BYTES[feat_dtype]
        self.max_batch_keys = max_batch_keys
        self.flags = int(flags)
        # WG_DSM_CSR_REPLICATED: this rank's slab holds the whole CSR (all num_nodes rows)
        self.csr_replicated = bool(self.flags & _lib.WG_DSM_CSR_REPLICATED)
        self._cb = _lib.ALLGATHER_FN(allgather) if allgather is not None else _lib.ALLGATHER_FN()
        d = _lib.WgDsmDesc(rank=rank, world_size=world_size, device=self.device.index, feat_dtype=DTYPE_CODE[feat_dtype],
                           num_nodes=num_nodes, local_num_edges=local_num_edges, feat_dim=feat_dim,
                           max_batch_keys=max_batch_keys, allgather=self._cb, ctx=None,
                           flags=self.flags, reserved=0)
        h = ctypes.c_void_p()
        check(lib().wg_dsm_create(ctypes.byref(d), ctypes.byref(h)))
        self.h = h
        self.gather_occupancy = 0
        # feature-row layout (wg_dsm_feat_layout): bytes [0, body_bytes) of a row in the feature
        # shard, the rest (split layout only) in the tail region
        bb, bp, tp, tpitch = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_void_p(), ctypes.c_int64()
        check(lib().wg_dsm_feat_layout(h, ctypes.byref(bb), ctypes.byref(bp), ctypes.byref(tp), ctypes.byref(tpitch)))
        self.body_bytes, self.tail_pitch, self._tail_ptr = bb.value, tpitch.value, tp.value

    # --- shard access
    def local_view(self):
        rp, col, feat = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
        nl, stride = ctypes.c_int64(), ctypes.c_int64()
        check(lib().wg_dsm_local_view(self.h, ctypes.byref(rp), ctypes.byref(col), ctypes.byref(feat),
                                      ctypes.byref(nl), ctypes.byref(stride)))
        n_local = nl.value
        _, e_local = self.shard_info(self.rank)
        csr_rows = self.num_nodes if self.csr_replicated else n_local
        row_ptr = device_view(rp.value, (csr_rows + 1,), torch.int64, self.device)
        col_dtype = torch.int32 if self.flags & _lib.WG_DSM_COL32 else torch.int64  # uint32 entries (< 2^31 here)
        colv = device_view(col.value, (e_local,), col_dtype, self.device)
        featv = device_view(feat.value, (n_local, stride.value), torch.uint8, self.device) if self.row_bytes else None
        return row_ptr, colv, featv

    def tail_view(self):
        """uint8 [n_local, tail_pitch] view of this rank's tail region (split layout), else None."""
        if not self.tail_pitch:
            return None
        n_local, _ = self.shard_info(self.rank)
        return device_view(self._tail_ptr, (n_local, self.tail_pitch), torch.uint8, self.device)

    def write_local_rows(self, rows_u8, start=0):
        """Write whole feature rows (uint8 [k, row_bytes], host or device) to local rows
        start .. start+k-1 of this rank's shard, honouring the row layout."""
        _, _, fv = self.local_view()
        src = rows_u8 if isinstance(rows_u8, torch.Tensor) else torch.from_numpy(np.ascontiguousarray(rows_u8))
        k, b = src.shape[0], self.body_bytes
        fv[start:start + k, :b].copy_(src[:, :b])
        if self.tail_pitch:
            self.tail_view()[start:start + k].copy_(src[:, b:self.row_bytes])

    def read_local_rows(self, local_rows):
        """Whole feature rows (uint8 [k, row_bytes], device) of the given local rows of this rank."""
        _, _, fv = self.local_view()
        body = fv[local_rows][:, :self.body_bytes]
        if not self.tail_pitch:
            return body
        return torch.cat([body, self.tail_view()[local_rows]], dim=1)

    def shard_info(self, r):
        nl, el = ctypes.c_int64(), ctypes.c_int64()
        check(lib().wg_dsm_shard_info(self.h, r, ctypes.byref(nl), ctypes.byref(el)))
        return nl.value, el.value

    def device_error(self, clear=True):
        c = ctypes.c_uint32()
        check(lib().wg_device_error(self.h, ctypes.byref(c), 1 if clear else 0))
        return c.value

    def chase(self, rank, span_bytes, accesses, stream=None):
        """Table-I-style dependent-load latency through rank's feature shard; returns ns/access."""
        sink = torch.zeros(1, dtype=torch.int64, device=self.device)
        s = stream or torch.cuda.current_stream(self.device)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        check(lib().wg_dsm_chase(self.h, rank, span_bytes, accesses, _ptr(sink), _stream(s)))
        e1.record(s)
        e1.synchronize()
        return e0.elapsed_time(e1) * 1e6 / accesses

    def reset_workspace(self, stream=None):
        check(lib().wg_dsm_reset_workspace(self.h, _stream(stream)))

    def set_stage_events(self, events):
        """Diagnostics: record these torch.cuda.Events after each kernel of the next ops
        (wg_dsm_set_stage_events); [] clears.  The events must have been recorded once (created)."""
        arr = (ctypes.c_void_p * max(len(events), 1))(*[e.cuda_event for e in events])
        check(lib().wg_dsm_set_stage_events(self.h, arr, len(events)))

    def unique_format(self):
        """Append Unique key-table format of this handle's workspace (wg_dsm_unique_format):
        WG_UNIQUE_WIDE / WG_UNIQUE_COMPACT / WG_UNIQUE_DIRECT."""
        f = ctypes.c_int32(0)
        check(lib().wg_dsm_unique_format(self.h, ctypes.byref(f), None))
        return f.value

    def hop_insert_pass(self):
        """True if wg_sample_hop runs a separate insert pass (wide key table); False if its sampler
        inserts the keys (wg_dsm_unique_format)."""
        f, ip = ctypes.c_int32(0), ctypes.c_int32(0)
        check(lib().wg_dsm_unique_format(self.h, ctypes.byref(f), ctypes.byref(ip)))
        return bool(ip.value)

    def debug_set_epoch(self, epoch):
        """Test hook: set the workspace's hash-table epoch (wg_dsm_debug_set_epoch)."""
        check(lib().wg_dsm_debug_set_epoch(self.h, int(epoch)))

    def destroy(self):
        if self.h is not None and self.h.value:
            check(lib().wg_dsm_destroy(self.h))
        self.h = None

    def fork(self, max_batch_keys=0):
        """Another handle on the same shards with its own workspace (wg_dsm_fork), for
        preparing independent batches concurrently on another stream."""
        f = DSM.__new__(DSM)
        f.__dict__.update({k: v for k, v in self.__dict__.items() if k != "h"})
        if max_batch_keys:
            f.max_batch_keys = max_batch_keys
        h = ctypes.c_void_p()
        check(lib().wg_dsm_fork(self.h, max_batch_keys, ctypes.byref(h)))
        f.h = h
        return f  # the fork starts with the parent's gather occupancy (copied by wg_dsm_fork)

    # --- the three ops --------------------------------------------------------
    def sample_neighbors(self, targets, fanout, seed, hop, n_targets_dev=None, seed_dev=None, out_row_ptr=None,
                         out_nbrs=None, out_pos=None, out_num_edges=None, cap=None, with_pos=False, stream=None):
        """Multi-GPU sampling op, one hop.  ``targets`` int64 cuda;
        ``cap`` = host capacity (default len(targets)); ``n_targets_dev`` optional
        device count.  Returns (row_ptr, nbrs, pos|None, num_edges_dev)."""
        cap = targets.numel() if cap is None else cap
        dev = self.device
        if out_row_ptr is None:
            out_row_ptr = torch.empty(cap + 1, dtype=torch.int64, device=dev)
        if out_nbrs is None:
            out_nbrs = torch.empty(max(cap * fanout, 1), dtype=torch.int64, device=dev)
        if with_pos and out_pos is None:
            out_pos = torch.empty(max(cap * fanout, 1), dtype=torch.int32, device=dev)
        if out_num_edges is None:
            out_num_edges = torch.empty(1, dtype=torch.int64, device=dev)
        check(lib().wg_sample_neighbors(self.h, _ptr(targets), cap, _ptr(n_targets_dev), fanout,
                                        ctypes.c_uint64(seed & ((1 << 64) - 1)), _ptr(seed_dev), hop,
                                        _ptr(out_row_ptr), _ptr(out_nbrs), _ptr(out_pos), _ptr(out_num_edges),
                                        _stream(stream)))
        return out_row_ptr, out_nbrs, out_pos, out_num_edges

    def append_unique(self, targets, nbrs, n_targets=None, n_nbrs=None, n_targets_dev=None, n_nbrs_dev=None,
                      out_unique=None, out_num_unique=None, out_sub_col=None, out_dup=None, with_dup=False,
                      stream=None):
        """Append Unique op.  Returns (U, num_unique_dev, sub_col, dup|None)."""
        nT = targets.numel() if n_targets is None else n_targets
        nE = nbrs.numel() if n_nbrs is None else n_nbrs
        dev = self.device
        if out_unique is None:
            out_unique = torch.empty(max(nT + nE, 1), dtype=torch.int64, device=dev)
        if out_num_unique is None:
            out_num_unique = torch.empty(1, dtype=torch.int64, device=dev)
        if out_sub_col is None:
            out_sub_col = torch.empty(max(nE, 1), dtype=torch.int32, device=dev)
        if with_dup and out_dup is None:
            out_dup = torch.empty(max(nT + nE, 1), dtype=torch.int32, device=dev)
        check(lib().wg_append_unique(self.h, _ptr(targets), nT, _ptr(n_targets_dev), _ptr(nbrs), nE,
                                     _ptr(n_nbrs_dev), _ptr(out_unique), _ptr(out_num_unique), _ptr(out_sub_col),
                                     _ptr(out_dup), _stream(stream)))
        return out_unique, out_num_unique, out_sub_col, out_dup

    def sample_hop(self, targets, fanout, seed, hop, n_targets_dev=None, seed_dev=None, out=None, cap=None,
                   with_pos=False, with_dup=False, stream=None, side_stream=None):
        """One fused hop = sample_neighbors + append_unique (same results; wg_sample_hop).
        ``out`` = dict of preallocated buffers (row_ptr, nbrs, pos, num_edges, unique,
        num_unique, sub_col, dup).  If ``side_stream`` is given the relabel runs there
        and the caller must wait for it before reading sub_col / dup."""
        cap = targets.numel() if cap is None else cap
        dev = self.device
        E = max(cap * fanout, 1)
        o = dict(out or {})
        i64 = dict(dtype=torch.int64, device=dev)
        i32 = dict(dtype=torch.int32, device=dev)
        o.setdefault("row_ptr", torch.empty(cap + 1, **i64))
        o.setdefault("nbrs", torch.empty(E, **i64))
        o.setdefault("pos", torch.empty(E, **i32) if with_pos else None)
        o.setdefault("num_edges", torch.empty(1, **i64))
        o.setdefault("unique", torch.empty(max(cap + cap * fanout, 1), **i64))
        o.setdefault("num_unique", torch.empty(1, **i64))
        o.setdefault("sub_col", torch.empty(E, **i32))
        o.setdefault("dup", torch.empty(max(cap + cap * fanout, 1), **i32) if with_dup else None)
        check(lib().wg_sample_hop(self.h, _ptr(targets), cap, _ptr(n_targets_dev), fanout,
                                  ctypes.c_uint64(seed & ((1 << 64) - 1)), _ptr(seed_dev), hop, _ptr(o["row_ptr"]),
                                  _ptr(o["nbrs"]), _ptr(o["pos"]), _ptr(o["num_edges"]), _ptr(o["unique"]),
                                  _ptr(o["num_unique"]), _ptr(o["sub_col"]), _ptr(o["dup"]), _stream(stream),
                                  _stream(side_stream) if side_stream is not None else None))
        return o

    def gather_rows(self, ids, cap, begin_dev, end_dev, out, stream=None):
        """Rows [*begin_dev, *end_dev) of ids -> the same rows of out (wg_gather_rows); out is
        uint8 [*, pitch] with pitch >= row_bytes (a pitched buffer moves 32 B vectors)."""
        pitch = out.stride(0) if out.dim() == 2 else 0
        check(lib().wg_gather_rows(self.h, _ptr(ids), cap, _ptr(begin_dev), _ptr(end_dev), _ptr(out), pitch,
                                   _stream(stream)))
        return out

    def set_gather_occupancy(self, blocks_per_sm):
        """Resident gather blocks per SM for this handle's gathers (0 = occupancy maximum);
        read at enqueue / capture time (wg_dsm_set_gather_occupancy)."""
        check(lib().wg_dsm_set_gather_occupancy(self.h, int(blocks_per_sm)))
        self.gather_occupancy = int(blocks_per_sm)

    def out_pitch(self):
        """Output row pitch that lets the gather move whole 32 B vectors (row bytes rounded up to 32).  Dense
        rows of 32k + 16 bytes also move as 32 B source pieces (stored as 16 B halves) and write 4 % fewer
        bytes, but measured slower in the throughput pass (profiles/r02/ab_log.md), so buffers are pitched."""
        return (self.row_bytes + 31) // 32 * 32

    def gather(self, ids, n_ids=None, n_ids_dev=None, out=None, stream=None):
        """Global gather: out[i] = feature row of ids[i] (uint8 rows)."""
        n = ids.numel() if n_ids is None else n_ids
        if out is None:
            out = torch.empty((max(n, 1), self.row_bytes), dtype=torch.uint8, device=self.device)
        check(lib().wg_gather(self.h, _ptr(ids), n, _ptr(n_ids_dev), _ptr(out), _stream(stream)))
        return out

    # --- filling helpers (setup; not on the hot path) ----------------------------
    def fill_from_global_csr(self, row_ptr, col):
        """Copy THIS rank's rows (v = rank, rank+W, ...) of a host CSR into its shard (every row
        with WG_DSM_CSR_REPLICATED)."""
        if self.csr_replicated:
            lrp, lcol = np.asarray(row_ptr, dtype=np.int64), np.asarray(col, dtype=np.int64)
        else:
            lrp, lcol = shard_csr(row_ptr, col, self.rank, self.world)
        rp, cv, _ = self.local_view()
        rp.copy_(torch.from_numpy(lrp))
        if len(lcol):
            cv.copy_(torch.from_numpy(lcol))

    def fill_features(self, rows_u8):
        """Copy this rank's feature rows (uint8 [n_local, row_bytes], host) into its shard."""
        self.write_local_rows(rows_u8, 0)


def shard_csr(row_ptr, col, rank, world):
    """Rows owned by ``rank`` under o(v) = v mod W, local row l(v) = v div W."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    n = len(row_ptr) - 1
    v = np.arange(rank, n, world, dtype=np.int64)
    starts, ends = row_ptr[v], row_ptr[v + 1]
    lens = ends - starts
    lrp = np.zeros(len(v) + 1, dtype=np.int64)
    lrp[1:] = np.cumsum(lens)
    idx = np.repeat(starts - lrp[:-1], lens) + np.arange(lrp[-1], dtype=np.int64)
    return lrp, np.asarray(col, dtype=np.int64)[idx]


def local_num_edges(row_ptr, rank, world):
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    n = len(row_ptr) - 1
    v = np.arange(rank, n, world, dtype=np.int64)
    return int((row_ptr[v + 1] - row_ptr[v]).sum())
