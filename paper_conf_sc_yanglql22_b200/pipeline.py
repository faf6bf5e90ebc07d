"""Multi-hop mini-batch preparation: "Multi-layer sub-graph sampling can be done by
simply stacking multiple single-layer sub-graph sampling", then
the global gather of the last frontier's features (L176).

All buffers are preallocated from host upper bounds (T_{h+1} = U_h <= min(n,
T_h (1 + M_h))) and every op reads the previous op's DEVICE count, so a whole batch
is enqueued without a host sync and can be captured once as a CUDA graph and
replayed with new seeds / rng_seed written into device buffers.
"""

import contextlib
import os

import torch

from .dsm import DSM

# NVTX ranges (host-side enqueue of every hop / gather, loader submit / collect) for nsys-style timelines;
# off unless WG_NVTX=1 in the environment at import (the ranges cost host time on the e2e path).
_NVTX = os.environ.get("WG_NVTX", "0") == "1"


@contextlib.contextmanager
def nvtx_range(name):
    if not _NVTX:
        yield
        return
    torch.cuda.nvtx.range_push(name)
    try:
        yield
    finally:
        torch.cuda.nvtx.range_pop()


def capacities(n, fanouts, max_seeds):
    T, E, U = [], [], []
    t = min(max_seeds, n)
    for m in fanouts:
        T.append(t)
        E.append(t * m)
        u = min(n, t + t * m)
        U.append(u)
        t = u
    return T, E, U


def required_keys(n, fanouts, max_seeds):
    T, E, _ = capacities(n, fanouts, max_seeds)
    return max(t + e for t, e in zip(T, E))


# Gather occupancy (resident gather blocks per SM, wg_dsm_set_gather_occupancy) for batches prepared
# several at a time on one GPU: a gather at full occupancy holds the whole register file and keeps
# the other streams' latency-bound hop kernels from overlapping it ("Concurrency").
THROUGHPUT_GATHER_OCCUPANCY = 1
EXCL_RING = 4     # scan buffers per DSM workspace (wg_sample_hop: join the side stream before a fifth hop)
PARAMS_RING = 64  # pinned staging slots for the per-batch scalars (batches enqueued ahead per pipeline)


class MiniBatchPipeline:
    def __init__(self, dsm: DSM, fanouts, max_seeds, with_pos=False, with_dup=False, fused=True,
                 incremental_gather=True, gather_priority=0, side_priority=0, gather_occupancy=None, x_pitch=None):
        self.dsm, self.fanouts, self.max_seeds = dsm, list(fanouts), max_seeds
        # None: use the handle's setting; an int: applied to this pipeline's gathers at enqueue
        self.gather_occupancy = gather_occupancy
        self.fused = fused
        self.side = torch.cuda.Stream(device=dsm.device, priority=side_priority) if fused else None
        # incremental gather: U_{h-1} is a prefix of U_h, so the feature rows of hop h's new nodes
        # are gathered on gside while hop h+1 samples; only the last hop's new rows remain at the end
        self.incremental = incremental_gather
        self.gside = torch.cuda.Stream(device=dsm.device, priority=gather_priority) if incremental_gather else None
        self.with_pos, self.with_dup = with_pos, with_dup
        dev = dsm.device
        self.T_cap, self.E_cap, self.U_cap = capacities(dsm.num_nodes, fanouts, max_seeds)
        if required_keys(dsm.num_nodes, fanouts, max_seeds) > dsm.max_batch_keys:
            raise ValueError("DSM workspace too small for this pipeline (max_batch_keys)")
        i64 = dict(dtype=torch.int64, device=dev)
        i32 = dict(dtype=torch.int32, device=dev)
        # the batch's inputs in ONE device buffer [n_seeds, rng_seed (uint64 bit pattern), seed ids...], so a
        # batch is written by one copy (set_inputs from host ids / set_inputs_packed); per-hop counts in one
        # [H, 2] buffer (one D2H copy)
        self.inbuf = torch.zeros(2 + max(self.max_seeds, 1), **i64)
        self.params = self.inbuf[0:2]
        self.n_seeds, self.rng_seed = self.inbuf[0:1], self.inbuf[1:2]
        self.seeds = self.inbuf[2:]
        # a ring of pinned staging buffers, so the host can enqueue many batches ahead without waiting
        self._params_host = torch.zeros((PARAMS_RING, self.inbuf.numel()), dtype=torch.int64, pin_memory=True)
        self._params_ev = [None] * PARAMS_RING
        self._params_next = 0
        self.counts_dev = torch.zeros((len(self.fanouts), 2), **i64)
        self.hops = []
        for h, m in enumerate(self.fanouts):
            T, E, U = self.T_cap[h], self.E_cap[h], self.U_cap[h]
            self.hops.append(dict(
                row_ptr=torch.zeros(T + 1, **i64), nbrs=torch.zeros(max(E, 1), **i64),
                pos=torch.zeros(max(E, 1), **i32) if with_pos else None,
                num_edges=self.counts_dev[h, 0:1], unique=torch.zeros(max(T + E, 1), **i64),
                num_unique=self.counts_dev[h, 1:2], sub_col=torch.zeros(max(E, 1), **i32),
                dup=torch.zeros(max(T + E, 1), **i32) if with_dup else None))
        # X is pitched to a 32 B multiple (DSM.out_pitch) so every row moves as whole 32 B vectors; X_rows is
        # the [U, row_bytes] view of the feature bytes (self.X[:, :row_bytes]).  x_pitch: another output
        # pitch (a multiple of 16 >= row_bytes, e.g. 400 = dense 400 B rows: 32 B loads, 16 B stores; A/B)
        pitch = dsm.out_pitch() if x_pitch is None else x_pitch
        self.X = torch.zeros((max(self.U_cap[-1], 1), pitch), dtype=torch.uint8, device=dev) \
            if dsm.row_bytes else None
        self.X_rows = self.X[:, :dsm.row_bytes] if self.X is not None else None
        self.graph = None

    # -- enqueue one batch (reads seeds / n_seeds / rng_seed from device buffers)
    def enqueue(self, stream=None, gather=True, gather_occupancy=None):
        """Enqueue every hop (fused wg_sample_hop: sample + append-unique; the
        relabel of each hop runs on a side stream, joined at the end) and, unless
        gather=False, the feature gather.  gather_occupancy (else the pipeline's) sets
        the gathers' blocks per SM for this enqueue only."""
        occ = self.gather_occupancy if gather_occupancy is None else gather_occupancy
        if occ is None or occ == self.dsm.gather_occupancy:
            return self._enqueue(stream, gather)
        prev = self.dsm.gather_occupancy
        self.dsm.set_gather_occupancy(occ)
        try:
            return self._enqueue(stream, gather)
        finally:
            self.dsm.set_gather_occupancy(prev)

    def _enqueue(self, stream=None, gather=True):
        d = self.dsm
        main = stream or torch.cuda.current_stream(d.device)
        if self.fused:
            self.side.wait_stream(main)
        tgt, tcap, tn = self.seeds, self.max_seeds, self.n_seeds
        incr = gather and self.incremental and self.X is not None
        prev_nu = None
        for h, m in enumerate(self.fanouts):
            b = self.hops[h]
            if self.fused and h and h % EXCL_RING == 0:
                # the workspace keeps a ring of EXCL_RING scan buffers read by the side-stream relabels:
                # hop h reuses hop h-EXCL_RING's buffer, so that relabel must be done (include/wg.h)
                main.wait_stream(self.side)
            if self.fused:
                with nvtx_range(f"wg.sample_hop h{h}"):
                    d.sample_hop(tgt, m, 0, h, n_targets_dev=tn, seed_dev=self.rng_seed, out=b, cap=tcap,
                                 stream=main, side_stream=self.side)
            else:
                d.sample_neighbors(tgt, m, 0, h, n_targets_dev=tn, seed_dev=self.rng_seed, out_row_ptr=b["row_ptr"],
                                   out_nbrs=b["nbrs"], out_pos=b["pos"], out_num_edges=b["num_edges"], cap=tcap,
                                   stream=main)
                d.append_unique(tgt, b["nbrs"], n_targets=tcap, n_nbrs=self.E_cap[h], n_targets_dev=tn,
                                n_nbrs_dev=b["num_edges"], out_unique=b["unique"], out_num_unique=b["num_unique"],
                                out_sub_col=b["sub_col"], out_dup=b["dup"], stream=main)
            if incr:  # rows [|U_{h-1}|, |U_h|) of X are final now
                self.gside.wait_stream(main)
                with nvtx_range(f"wg.gather_rows h{h}"):
                    d.gather_rows(b["unique"], self.U_cap[h], prev_nu, b["num_unique"], self.X, stream=self.gside)
                prev_nu = b["num_unique"]
            tgt, tcap, tn = b["unique"], self.U_cap[h], b["num_unique"]
        if gather and self.X is not None and not incr:
            self.enqueue_gather(main)
        if self.fused:
            main.wait_stream(self.side)
        if incr:
            main.wait_stream(self.gside)

    def enqueue_gather(self, stream=None):
        last = self.hops[-1]
        self.dsm.gather_rows(last["unique"], self.U_cap[-1], None, last["num_unique"], self.X, stream=stream)

    def set_inputs(self, seeds: torch.Tensor, rng_seed: int, stream=None):
        """Write this batch's seed nodes (host or device int64) and (n_seeds, rng_seed) into the pipeline's
        input buffer, stream-ordered, no kernel: host ids are packed with the scalars into a pinned staging
        slot and moved by ONE H2D copy; device ids take a D2D copy plus a 16 B H2D of the scalars."""
        n = seeds.numel()
        if n > self.max_seeds:
            raise ValueError("too many seeds")
        s = stream or torch.cuda.current_stream()
        k = self._params_next
        self._params_next = (k + 1) % PARAMS_RING
        if self._params_ev[k] is not None:
            self._params_ev[k].synchronize()   # that slot's earlier copy has read it (PARAMS_RING batches ago)
        else:
            self._params_ev[k] = torch.cuda.Event()
        stage = self._params_host[k]
        stage[0] = n
        stage[1] = to_i64(rng_seed)
        with torch.cuda.stream(s):
            if seeds.is_cuda:
                self.seeds[:n].copy_(seeds, non_blocking=True)
                self.params.copy_(stage[:2], non_blocking=True)
            else:
                stage[2:2 + n].copy_(seeds)
                self.inbuf[:2 + n].copy_(stage[:2 + n], non_blocking=True)
            self._params_ev[k].record(s)

    def set_inputs_packed(self, packed: torch.Tensor, stream=None):
        """One D2D copy of a device int64 buffer already laid out as the input buffer: [n_seeds, rng_seed,
        seed ids...] (pack_inputs); n_seeds must equal packed.numel() - 2."""
        if packed.numel() - 2 > self.max_seeds or packed.numel() < 2:
            raise ValueError("packed inputs do not fit this pipeline")
        with torch.cuda.stream(stream or torch.cuda.current_stream()):
            self.inbuf[:packed.numel()].copy_(packed, non_blocking=True)

    def run(self, seeds, rng_seed, stream=None):
        self.set_inputs(seeds, rng_seed, stream)
        if self.graph is not None:
            self.graph.replay()
        else:
            self.enqueue(stream)

    def capture(self):
        """Capture enqueue() as one CUDA graph (call after a warm-up run)."""
        g = torch.cuda.CUDAGraph()
        s = torch.cuda.Stream(device=self.dsm.device)
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.graph(g, stream=s):
            self.enqueue()
        torch.cuda.current_stream().wait_stream(s)
        self.graph = g
        return g

    # -- results (host sync)
    def counts(self):
        out = []
        for b in self.hops:
            out.append((int(b["num_edges"].item()), int(b["num_unique"].item())))
        return out

    def result(self, h):
        """Host copies of hop h's outputs, trimmed to the device counts."""
        b = self.hops[h]
        nT = int(self.n_seeds.item()) if h == 0 else int(self.hops[h - 1]["num_unique"].item())
        e, u = int(b["num_edges"].item()), int(b["num_unique"].item())
        r = dict(row_ptr=b["row_ptr"][: nT + 1].cpu().numpy(), nbrs=b["nbrs"][:e].cpu().numpy(),
                 unique=b["unique"][:u].cpu().numpy(), sub_col=b["sub_col"][:e].cpu().numpy())
        if b["pos"] is not None:
            r["pos"] = b["pos"][:e].cpu().numpy()
        if b["dup"] is not None:
            r["dup"] = b["dup"][:u].cpu().numpy()
        return r

    def features(self):
        u = int(self.hops[-1]["num_unique"].item())
        return self.X_rows[:u].contiguous().cpu().numpy()


def pack_inputs(seeds, rng_seed: int, device=None) -> torch.Tensor:
    """[n_seeds, rng_seed, seed ids...] as one int64 tensor (for MiniBatchPipeline.set_inputs_packed)."""
    s = torch.as_tensor(seeds, dtype=torch.int64).reshape(-1).cpu()
    head = torch.tensor([s.numel(), to_i64(rng_seed)], dtype=torch.int64)
    out = torch.cat([head, s])
    return out.to(device) if device is not None else out


def to_i64(x: int) -> int:
    x &= (1 << 64) - 1
    return x - (1 << 64) if x >= (1 << 63) else x


class PreparedBatch:
    """One prepared mini-batch handed out by MiniBatchLoader: host-side per-hop counts and
    DEVICE views of the pipeline slot's buffers (valid until the next batch is requested)."""

    def __init__(self, index, pipe, counts, n_seeds):
        self.index, self.pipe, self.n_seeds = index, pipe, n_seeds
        self.counts = counts          # [(num_edges, num_unique)] per hop, host ints

    def hop(self, h):
        """Hop h's sub-graph: row_ptr [T_h+1], nbrs / sub_col [E_h], unique [U_h] (device views)."""
        b = self.pipe.hops[h]
        nT = self.n_seeds if h == 0 else self.counts[h - 1][1]
        e, u = self.counts[h]
        return dict(row_ptr=b["row_ptr"][: nT + 1], nbrs=b["nbrs"][:e], sub_col=b["sub_col"][:e],
                    unique=b["unique"][:u], pos=None if b["pos"] is None else b["pos"][:e],
                    dup=None if b["dup"] is None else b["dup"][:u])

    @property
    def X(self):
        """Gathered feature bytes [U_{H-1}, row_bytes] (uint8 view, rows in unique order)."""
        return self.pipe.X_rows[: self.counts[-1][1]]


class MiniBatchLoader:
    """Pipelined mini-batch preparation: `depth` independent MiniBatchPipelines (one DSM
    workspace fork and one stream each) prepare consecutive batches concurrently, so the
    latency-bound hops of one batch overlap the bandwidth-bound gather of another.

    Every batch is: H2D of its seed ids (pinned host or device int64) and rng_seed, the
    captured batch graph (all hops + incremental gather), and a D2H of its per-hop counts
    into pinned memory.  `__call__(batches)` yields PreparedBatch objects in submission
    order, keeping up to `depth` batches in flight; a slot is reused only after the
    consumer's stream has passed the point where the batch was handed out."""

    def __init__(self, dsm: DSM, fanouts, max_seeds, depth=8, with_pos=False, with_dup=False, graphs=True,
                 gather_occupancy="auto"):
        self.depth = max(1, depth)
        self.handles = [dsm] + [dsm.fork() for _ in range(self.depth - 1)]
        if gather_occupancy == "auto":  # throughput mode when several batches share the GPU
            gather_occupancy = THROUGHPUT_GATHER_OCCUPANCY if self.depth >= 4 else None
        self.pipes = [MiniBatchPipeline(h, fanouts, max_seeds, with_pos=with_pos, with_dup=with_dup,
                                        gather_occupancy=gather_occupancy) for h in self.handles]
        dev = dsm.device
        self.streams = [torch.cuda.Stream(device=dev) for _ in range(self.depth)]
        self.done = [torch.cuda.Event() for _ in range(self.depth)]
        self.released = [None] * self.depth        # event recorded on the consumer stream at hand-out
        self.counts = [torch.zeros((len(fanouts), 2), dtype=torch.int64, pin_memory=True)
                       for _ in range(self.depth)]
        self.n_seeds = [0] * self.depth
        self.use_graphs = graphs
        self.graphs = [None] * self.depth
        self.warm = [0] * self.depth
        self.next_slot = 0

    def submit(self, seeds, rng_seed):
        """Enqueue one batch on the next slot; returns the slot index (stream-ordered, no sync)."""
        with nvtx_range("wg.loader.submit"):
            return self._submit(seeds, rng_seed)

    def _submit(self, seeds, rng_seed):
        j = self.next_slot
        self.next_slot = (j + 1) % self.depth
        pl, st = self.pipes[j], self.streams[j]
        if self.released[j] is not None:
            st.wait_event(self.released[j])        # the consumer is done with the slot's last batch
            self.released[j] = None
        self.n_seeds[j] = seeds.numel()
        with torch.cuda.stream(st):
            pl.set_inputs(seeds, rng_seed, st)
            if self.graphs[j] is not None:
                self.graphs[j].replay()
            else:
                pl.enqueue(st)
                self.warm[j] += 1
            self.counts[j].copy_(pl.counts_dev, non_blocking=True)  # every hop's (edges, unique): one D2H
            self.done[j].record(st)
        if self.use_graphs and self.graphs[j] is None and self.warm[j] >= 1:
            self._capture(j)
        return j

    def _capture(self, j):
        st = self.streams[j]
        st.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            self.pipes[j].enqueue(st)
        self.graphs[j] = g

    def collect(self, j, index=0):
        """Wait (host) for slot j's batch and hand it out (call release(j) when the consumer's
        work on it has been enqueued)."""
        with nvtx_range("wg.loader.collect"):
            self.done[j].synchronize()
        counts = [(int(e), int(u)) for e, u in self.counts[j].tolist()]
        return PreparedBatch(index, self.pipes[j], counts, self.n_seeds[j])

    def release(self, j):
        """The slot may be refilled once the consumer stream reaches this point."""
        ev = torch.cuda.Event()
        ev.record(torch.cuda.current_stream(self.pipes[j].dsm.device))
        self.released[j] = ev

    def __call__(self, batches):
        """batches: iterable of (seed ids int64 tensor, rng_seed).  Yields PreparedBatch in order;
        a batch's buffers stay valid until the next batch is requested (its slot is released then,
        stream-ordered after whatever the consumer enqueued on the current stream)."""
        pending = []
        for i, (s, r) in enumerate(batches):
            if len(pending) == self.depth:
                k, j = pending.pop(0)
                yield self.collect(j, k)
                self.release(j)
            pending.append((i, self.submit(s, r)))
        for k, j in pending:
            yield self.collect(j, k)
            self.release(j)

    def device_error(self):
        err = 0
        for h in self.handles:
            err |= h.device_error()
        return err

    def close(self):
        torch.cuda.synchronize()
        self.graphs = [None] * self.depth
        for h in self.handles[1:]:
            h.destroy()
        self.handles = self.handles[:1]
