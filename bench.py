#!/usr/bin/env python
"""Benchmark of the mini-batch preparation hot path (BASELINE.json metric: seed
nodes/s sampled+gathered per box; gather GB/s vs the HBM/NVLink roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config products]
    torchrun --nproc-per-node N bench.py --gpus N ...       (one rank per GPU)
    python bench.py --impl reference ...                    (the CPU oracle arm)

A step = one mini-batch of `seeds_per_batch` seeds per GPU through every hop of
sampling + append-unique and the final feature gather.  The
whole step is captured as two CUDA graphs (prep, gather) and replayed; each rank
runs its own batches (b = r mod W) against the shared DSM (weak scaling).
"""

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="products", choices=["tiny", "products", "papers100m", "mag240m"])
    ap.add_argument("--impl", default="wg", choices=["wg", "reference"])
    ap.add_argument("--no-flush", action="store_true", help="do not flush L2 between steps")
    ap.add_argument("--no-graph", action="store_true", help="launch ops eagerly instead of graph replay")
    ap.add_argument("--cpu-sample-s", type=float, default=12.0, help="target seconds of oracle work (cpu_baseline)")
    ap.add_argument("--e2e-steps", type=int, default=20)
    ap.add_argument("--concurrency", type=int, default=8, help="independent batches in flight per GPU (streams)")
    ap.add_argument("--out", default=None, help="also append the JSON line to this file")
    ap.add_argument("--sweep", action="store_true", help="config 4: feature-gather sweep over row sizes")
    ap.add_argument("--sweep-rows", type=int, default=100_000_000)
    ap.add_argument("--sweep-ids", type=int, default=1_000_000)
    ap.add_argument("--sweep-cells", default=None, help="comma list of dtype:dim cells (default: the whole grid)")
    ap.add_argument("--latency", action="store_true", help="Table I analogue: dependent-load latency vs span")
    ap.add_argument("--layer", action="store_true", help="NEXT #2: g-SpMM mean aggregation on a prepared batch")
    ap.add_argument("--pass-b", default="both", choices=["both", "prep", "gather"],
                    help="diagnostics: run only the prep or only the gather in the throughput pass")
    ap.add_argument("--compare-gather", action="store_true", help="NEXT #1: P2P vs distributed-memory gather")
    ap.add_argument("--gather-occupancy", type=int, default=None,
                    help="gather blocks per SM in the throughput pass (default: pipeline.THROUGHPUT_GATHER_OCCUPANCY "
                         "when more than 3 batches are in flight; 0 = occupancy maximum)")
    ap.add_argument("--placement", default="dsm", choices=["dsm", "replicas"],
                    help="dsm (default, the paper's method): graph + features row-sharded over the W GPUs, remote "
                         "rows read over NVLink; replicas (SURVEY 8(e) lever, labelled): every GPU holds the whole "
                         "graph + table (a W=1 DSM each) when it fits in its HBM, no NVLink traffic")
    ap.add_argument("--chase-accesses", type=int, default=100_000)
    return ap.parse_args()


METRIC = "seed nodes/sec sampled+gathered per box"
UNIT = "seeds/s"


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """SM clock and clock-event (throttle) reasons sampled DURING the timed region: NVML polled every
    5 ms from a thread (nvidia-smi -lms 50 as a fallback)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.rows = []
        self.proc = None
        self.nv = None
        self.stop_ev = threading.Event()

    def start(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.gpu)
            self.nv, self.h = nv, h
            self.max_sm = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return
        except Exception:
            self.nv = None
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _poll(self):
        nv = self.nv
        while not self.stop_ev.is_set():
            try:
                sm = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.rows.append((sm, rs))
            except Exception:
                pass
            time.sleep(0.005)

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.nv is not None:
            self.stop_ev.set()
            self.t.join(timeout=2)
            nv = self.nv
            bits = {"hw_slowdown": nv.nvmlClocksEventReasonHwSlowdown,
                    "hw_thermal_slowdown": nv.nvmlClocksEventReasonHwThermalSlowdown,
                    "sw_thermal_slowdown": nv.nvmlClocksEventReasonSwThermalSlowdown,
                    "sw_power_cap": nv.nvmlClocksEventReasonSwPowerCap}
            reasons = sorted({k for _, r in self.rows for k, b in bits.items() if r & b})
            sm = [float(x) for x, _ in self.rows]
            return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": float(self.max_sm),
                    "reasons": reasons, "samples": len(sm), "source": "nvml, 5 ms"}
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm = [float(r[1]) for r in self.rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            if len(r) >= 9:
                for k, nm in enumerate(names):
                    if r[5 + k].lower() == "active":
                        reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm), "source": "nvidia-smi, 50 ms"}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


# ----------------------------------------------------------------------------- oracle arm
def run_oracle(preset, batches, sample_s, rank=0, world=1):
    """Time the CPU oracle (as it stands, single-threaded) on whole batches of the
    same workload; returns (seeds/s, seconds of oracle work, batches done, cores)."""
    import contextlib

    import oracle
    from paper_conf_sc_yanglql22_b200 import loader
    from synth import presets, seeds
    os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
    rows = loader.host_row_provider(preset.graph())
    feats = loader.host_feat_provider(preset)
    spent = [0.0]

    @contextlib.contextmanager
    def timer():
        t = time.perf_counter()
        yield
        spent[0] += time.perf_counter() - t
    done = 0
    for b in batches:
        S = seeds.seed_nodes(preset.n, preset.seeds_per_batch, presets.SEED_BASE, b)
        oracle.minibatch(rows, feats, S, preset.fanouts, seeds.rng_seed(presets.RNG_BASE, b), timer=timer)
        done += 1
        if spent[0] >= sample_s:
            break
    return done * preset.seeds_per_batch / spent[0], spent[0], done, len(os.sched_getaffinity(0))


def bench_reference(args):
    from synth import presets
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    p = presets.get(args.config)
    per_step = []
    total_s = 0.0
    for k in range(args.warmup + args.steps):
        v, s, done, cores = run_oracle(p, [k], 0.0)
        if k >= args.warmup:
            per_step.append(s)
            total_s += s
    value = args.steps * p.seeds_per_batch / total_s
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total_s / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64+fp32-bytes",
            "data": "synthetic", "config": workload_config(p, 1),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": f"{args.steps} whole batches of {p.seeds_per_batch} seeds "
                                       f"(fanout {p.fanouts} + gather), rows regenerated per hop (untimed)"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line, args)


# The paper's own numbers (DGX-A100 = 8 x A100 on NVSwitch, NVLink3 300 GB/s per direction):
# context next to ours, never the target.
PAPER_CONTEXT = {
    "hardware": "DGX-A100 (8x A100 80GB, NVSwitch, NVLink3 300 GB/s/dir), CUDA 11.4",
    "dsm_random_gather_busbw_gbs_ge128B": 230, "dsm_random_gather_busbw_frac_of_nvlink": 0.77,
    "p2p_dependent_load_latency_us_8_128GB": [1.35, 1.56],
    "epoch_speedup_vs_dgl_max": 57.32, "epoch_speedup_vs_pyg_max": 242.98,
    "ogbn_products_graphsage_epoch_s": {"wholegraph": 0.99, "dgl": 30.8, "pyg": 228.96},
    "seed_nodes_per_s": None,
    "note": "PAPER.md L5, L66-80, L266, L272-275; end-to-end training epochs, not this metric (the paper "
            "reports no seeds/s); context only",
}


def workload_config(p, W, flushed=True, placement="dsm"):
    par = (f"dsm-w{W} (row-sharded CSR+features, P2P loads, no hot-path collective)" if placement == "dsm" else
           f"replicas-x{W} (SURVEY 8(e) lever: whole graph + table on every GPU, no NVLink, no hot-path collective)")
    return {"workload": p.name, "nodes": p.n, "csr_entries_target": p.target_e, "fanouts": p.fanouts,
            "seeds_per_gpu": p.seeds_per_batch, "features": f"{p.feat_dim}x{p.feat_dtype}",
            "parallelism": par,
            "l2": "flushed between steps (512 MB write outside the events)" if flushed else "not flushed",
            "note": p.note}



def workload_descriptors(dsm, pipe, seeds_dev, rngs, nb=20):
    """SURVEY 8(d) workload descriptors (generator properties that drive the numbers): this rank's
    out-degree distribution, and the share of gathered rows that falls on the top 1 % most-gathered
    rows over nb batches (outside every timed region)."""
    import torch
    rp, _, _ = dsm.local_view()
    deg = (rp[1:] - rp[:-1]).double()
    lg = torch.floor(torch.log2(deg.clamp(min=1))).long()
    hist = torch.bincount(lg, minlength=18).tolist()
    cnt = torch.zeros(dsm.num_nodes, dtype=torch.int32, device=rp.device)
    tot = 0
    for k in range(min(nb, len(seeds_dev))):
        pipe.run(seeds_dev[k], rngs[k])
        u = pipe.hops[-1]["unique"][: int(pipe.hops[-1]["num_unique"].item())]
        cnt.index_add_(0, u, torch.ones_like(u, dtype=torch.int32))
        tot += u.numel()
    top = torch.topk(cnt, max(1, dsm.num_nodes // 100)).values.sum().item()
    q = torch.quantile(deg[: 1 << 24], torch.tensor([0.5, 0.99], dtype=torch.float64, device=deg.device)).tolist()
    return {"degree_mean": float(deg.mean()), "degree_max": int(deg.max()), "degree_p50": q[0], "degree_p99": q[1],
            "degree_log2_hist": hist, "top1pct_rows_share_of_gathered": top / max(tot, 1),
            "batches_for_share": min(nb, len(seeds_dev))}

def stage_breakdown(pipe, seeds_dev, rngs, flush, nb=20):
    """SURVEY 8(d) per-stage device times of one batch (outside every timed region): each hop's
    fused op (sample + append-unique + relabel, all on one stream here) and the whole gather,
    with a CUDA event after every op, eager launches, L2 flushed before each batch; medians."""
    import torch
    st = torch.cuda.current_stream()
    H = len(pipe.fanouts)
    names = [f"hop{h}" for h in range(H)] + ["gather"]
    acc = {n: [] for n in names}
    for b in range(nb + 2):
        pipe.set_inputs(seeds_dev[b % len(seeds_dev)], rngs[b % len(rngs)])
        if flush is not None:
            flush.fill_(b & 0xFF)
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(H + 2)]
        evs[0].record(st)
        tgt, tcap, tn = pipe.seeds, pipe.max_seeds, pipe.n_seeds
        for h, m in enumerate(pipe.fanouts):
            bb = pipe.hops[h]
            pipe.dsm.sample_hop(tgt, m, 0, h, n_targets_dev=tn, seed_dev=pipe.rng_seed, out=bb, cap=tcap, stream=st)
            evs[h + 1].record(st)
            tgt, tcap, tn = bb["unique"], pipe.U_cap[h], bb["num_unique"]
        pipe.enqueue_gather(st)
        evs[H + 1].record(st)
        torch.cuda.synchronize()
        if b >= 2:
            for i, n in enumerate(names):
                acc[n].append(evs[i].elapsed_time(evs[i + 1]))
    out = {n: statistics.median(v) for n, v in acc.items()}
    out["note"] = ("median ms per stage of one batch (eager launches, event after every op, L2 flushed per "
                   "batch; hop h = wg_sample_hop: sample + insert + flag-scan + relabel)")
    return out


def emit(line, args):
    s = json.dumps(line)
    print(s, flush=True)
    if args.out:
        with open(args.out, "a") as f:
            f.write(s + "\n")


# ----------------------------------------------------------------------------- GPU arm
def bench_wg(args):
    import torch
    import torch.distributed as dist

    import paper_conf_sc_yanglql22_b200 as pkg
    from paper_conf_sc_yanglql22_b200 import loader
    from synth import presets, seeds

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ndev = torch.cuda.device_count()
    torch.cuda.set_device(local % ndev)
    dev = torch.device("cuda", local % ndev)
    ag = None
    backend = None
    if world > 1:
        # one rank per GPU over NCCL; if ranks share a GPU (a test box with fewer GPUs than ranks)
        # NCCL refuses, so the setup-time handle exchange falls back to gloo (never on the hot path)
        backend = "nccl" if ndev >= int(os.environ.get("LOCAL_WORLD_SIZE", world)) else "gloo"
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
        ag = pkg.TorchDistAllgather(device=dev)
    local = local % ndev
    p = presets.get(args.config)
    S = p.seeds_per_batch
    P = max(1, args.concurrency)
    t0 = time.perf_counter()
    if args.placement == "replicas":  # every rank its own whole copy (a W=1 DSM); batches still b = r mod W
        dsm, info = loader.build_dsm(p, rank=0, world=1, device=local, allgather=None)
    else:
        dsm, info = loader.build_dsm(p, rank=rank, world=world, device=local, allgather=ag)
    setup_s = time.perf_counter() - t0
    # P independent batch pipelines on P streams; pipeline j > 0 runs on a workspace fork of the DSM
    handles = [dsm] + [dsm.fork() for _ in range(P - 1)]
    pipes = [pkg.MiniBatchPipeline(h, p.fanouts, S) for h in handles]
    streams = [torch.cuda.Stream(device=dev) for _ in range(P)]
    n_single = args.warmup + args.steps
    n_conc = args.warmup + args.steps * P
    my_batches = [k * world + rank for k in range(n_single + n_conc)]
    seeds_dev = [torch.from_numpy(seeds.seed_nodes(p.n, S, presets.SEED_BASE, b)).to(dev) for b in my_batches]
    rngs = [seeds.rng_seed(presets.RNG_BASE, b) for b in my_batches]
    flush = None if args.no_flush else torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    # warm-up (eager), then capture each pipeline as two graphs (prep, gather) on its stream
    for k in range(args.warmup):
        for pl in pipes:
            pl.run(seeds_dev[k], rngs[k])
    torch.cuda.synchronize()
    from paper_conf_sc_yanglql22_b200 import pipeline as pipemod
    occ_b = args.gather_occupancy
    if occ_b is None:
        occ_b = pipemod.THROUGHPUT_GATHER_OCCUPANCY if P >= 4 else 0
    graphs, full_graphs, tput_graphs = [], [], []
    for pl, st in zip(pipes, streams):
        if args.no_graph:
            graphs.append((None, None))
            full_graphs.append(None)
            tput_graphs.append(None)
            continue
        st.wait_stream(torch.cuda.current_stream())
        gp, gg, gf = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
        with torch.cuda.graph(gp, stream=st):      # pass A: hops only ...
            pl.enqueue(gather=False)
        with torch.cuda.graph(gg, stream=st):      # ... then the whole gather (the roofline kernel)
            pl.enqueue_gather()
        with torch.cuda.graph(gf, stream=st):      # pass A': the batch as shipped (incremental gather)
            pl.enqueue(gather=True, gather_occupancy=0)
        gb = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gb, stream=st):      # pass B: the same with the throughput gather occupancy
            pl.enqueue(gather=True, gather_occupancy=occ_b)
        graphs.append((gp, gg))
        full_graphs.append(gf)
        tput_graphs.append(gb)
    torch.cuda.synchronize()

    def launch(j, k, st):
        """batch k on pipeline j, stream st (inputs already resident in HBM)."""
        pl, (gp, gg) = pipes[j], graphs[j]
        with torch.cuda.stream(st):
            pl.set_inputs(seeds_dev[k], rngs[k])
            if gp is not None:
                gp.replay()
            else:
                pl.enqueue(gather=False)
        return pl, gg

    def gather(j, st):
        pl, (gp, gg) = pipes[j], graphs[j]
        with torch.cuda.stream(st):
            if gg is not None:
                gg.replay()
            else:
                pl.enqueue_gather()

    def whole(j, k, st, tput=False):
        """batch k through pipeline j as one graph: hops + incremental gather (tput: the gathers at
        the throughput occupancy, for batches prepared concurrently)."""
        pl = pipes[j]
        g = (tput_graphs if tput else full_graphs)[j]
        with torch.cuda.stream(st):
            pl.set_inputs(seeds_dev[k], rngs[k])
            if g is not None:
                g.replay()
            else:
                pl.enqueue(gather_occupancy=occ_b if tput else 0)

    for k in range(args.warmup):     # warm the graphs
        for j in range(P):
            launch(j, k, streams[j])
            gather(j, streams[j])
            whole(j, k, streams[j])
            whole(j, k, streams[j], tput=True)
    torch.cuda.synchronize()
    for h in handles:
        err = h.device_error()
        assert err == 0, f"device error {err:#x} during warm-up"

    main = torch.cuda.current_stream()
    clocks = ClockSampler(local)

    # ---- pass A: one batch at a time (single-batch latency + the gather roofline)
    evA = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    rows_gathered = torch.zeros(args.steps, dtype=torch.int64, device=dev)
    hop_counts = torch.zeros((args.steps, len(p.fanouts), 2), dtype=torch.int64, device=dev)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if rank == 0 or world == 1:
        clocks.start()
    wall0 = time.perf_counter()
    for i in range(args.steps):
        k = args.warmup + i
        if flush is not None:
            flush.fill_(i & 0xFF)
        evA[i][0].record(main)
        pl, _ = launch(0, k, main)
        evA[i][1].record(main)
        gather(0, main)
        evA[i][2].record(main)
        rows_gathered[i:i + 1].copy_(pl.hops[-1]["num_unique"])
        for h, b in enumerate(pl.hops):
            hop_counts[i, h, 0:1].copy_(b["num_edges"])
            hop_counts[i, h, 1:2].copy_(b["num_unique"])
    torch.cuda.synchronize()
    step_ms = [evA[i][0].elapsed_time(evA[i][2]) for i in range(args.steps)]
    gather_ms = [evA[i][1].elapsed_time(evA[i][2]) for i in range(args.steps)]
    # pass A': one batch at a time through the shipped graph (hops + incremental gather)
    evW = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(args.steps)]
    for i in range(args.steps):
        if flush is not None:
            flush.fill_(i & 0xFF)
        evW[i][0].record(main)
        whole(0, args.warmup + i, main)
        evW[i][1].record(main)
    torch.cuda.synchronize()
    whole_ms = [evW[i][0].elapsed_time(evW[i][1]) for i in range(args.steps)]

    # ---- pass B: the throughput number.  P batch pipelines run continuously on P streams (pipeline j
    # prepares batches j, j+P, ...; its next batch starts when its previous gather is done, the other
    # pipelines fill the gaps).  K steps of P batches are timed as one region (events on the main
    # stream, barrier + synchronize on both sides); no L2 flush inside it: the inputs (graph + feature
    # table, ~2 GB) are far larger than the 126 MB L2 and every batch is new.
    evB = [torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    evB[0].record(main)
    for j in range(P):
        streams[j].wait_stream(main)
    for i in range(args.steps):
        for j in range(P):
            if args.pass_b == "both":
                whole(j, n_single + args.warmup + i * P + j, streams[j], tput=True)
                continue
            if args.pass_b != "gather":
                launch(j, n_single + args.warmup + i * P + j, streams[j])
            if args.pass_b != "prep":
                gather(j, streams[j])
    for j in range(P):
        main.wait_stream(streams[j])
    evB[1].record(main)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    conc_ms = [evB[0].elapsed_time(evB[1])]
    for h in handles:
        err = h.device_error()
        assert err == 0, f"device error {err:#x} in the timed region"

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    dev_s_single = max_over_ranks(sum(step_ms) / 1e3)
    dev_s_conc = max_over_ranks(sum(conc_ms) / 1e3)
    dev_s_whole = max_over_ranks(statistics.mean(whole_ms) / 1e3)  # collective: every rank, outside rank-0 code
    value_single = world * S * args.steps / dev_s_single
    value_conc = world * S * P * args.steps / dev_s_conc
    rb = dsm.row_bytes
    rows = rows_gathered.cpu().numpy()
    hc = hop_counts.cpu().numpy()
    gather_s = sum(gather_ms) / 1e3
    # roofline of the gather: t_roof = max(2RB / HBM, (W-1)/W * RB / NVLink); at W=1 every
    # byte is local HBM (read + write); at W>1 the (W-1)/W remote share crosses NVLink (770 GB/s measured
    # peer bandwidth per direction, B200_PROFILING.md; 900 nominal) and bounds the kernel.
    peak, peak_src = peaks()
    hbm_bytes = float(2 * rows.sum() * rb)
    wd = world if args.placement == "dsm" else 1  # replicas: every row is local
    nvl_bytes = float((wd - 1) / wd * rows.sum() * rb)
    t_hbm = hbm_bytes / (peak * 1e9)
    t_nvl = nvl_bytes / 770e9
    shared_gpu = world > 1 and torch.cuda.device_count() < world  # test box: "remote" rows are local HBM
    if t_nvl > t_hbm and not shared_gpu:
        bound, alg_bytes, peak_used, peak_src_used = "nvlink", nvl_bytes, 770.0, \
            "measured peer copy BW per direction (B200_PROFILING.md; 900 nominal)"
    else:
        bound, alg_bytes, peak_used, peak_src_used = "hbm", hbm_bytes, peak, peak_src
    achieved = alg_bytes / gather_s / 1e9

    # ---- e2e through the public API (MiniBatchLoader): every batch = H2D of its seeds from pinned host
    # memory + the batch graph + D2H of its per-hop counts, P batches in flight (as pass B), host-timed
    # from the first submit to the last batch handed out
    loader_ = pkg.MiniBatchLoader(dsm, p.fanouts, S, depth=P, gather_occupancy=occ_b)
    host_seeds = [seeds_dev[k % n_single].cpu().pin_memory() for k in range(args.e2e_steps * P)]
    warm = [(host_seeds[k % len(host_seeds)], rngs[k % n_single]) for k in range(2 * P)]
    for _ in loader_(warm):
        pass
    torch.cuda.synchronize()
    todo = [(host_seeds[k], rngs[(n_single + k) % len(rngs)]) for k in range(args.e2e_steps * P)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t = time.perf_counter()
    e2e_rows = 0
    for pb in loader_(todo):
        e2e_rows += pb.counts[-1][1]
    e2e_s = time.perf_counter() - t
    assert loader_.device_error() == 0
    e2e_val = world * S * len(todo) / max_over_ranks(e2e_s)
    e2e_d2h = len(p.fanouts) * 2 * 8
    loader_.close()

    wdesc = workload_descriptors(dsm, pipes[0], seeds_dev, rngs) if rank == 0 else {}
    stages = stage_breakdown(pipes[0], seeds_dev, rngs, flush) if rank == 0 else {}
    line = None
    if rank == 0:
        cpu = None
        if world == 1 and args.cpu_sample_s > 0:
            v, s_spent, done, cores = run_oracle(p, range(10_000, 10_100), args.cpu_sample_s)
            cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
                   "sample": f"{done} whole batches of {S} seeds (fanout {p.fanouts} + gather) of the same workload, "
                             f"{s_spent:.1f} s of single-threaded oracle work (row regeneration untimed)"}
        cfg = workload_config(p, world, flush is not None, args.placement)
        cfg["concurrent_batches_per_gpu"] = P
        cfg["gather_blocks_per_sm_throughput_pass"] = occ_b or "occupancy max"
        cfg["l2"] = ("pass A (single batch, roofline): L2 flushed between batches; pass B (value): continuous, "
                     "inputs (2 GB graph + features) >> 126 MB L2, every batch new")
        line = {
            "metric": METRIC, "value": value_conc, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * dev_s_conc / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64 ids + fp32 feature bytes",
            "data": "synthetic (seeded power-law graph + procedural features, see DESIGN.md)",
            "config": cfg,
            "single_batch": {"value": world * S / dev_s_whole, "unit": UNIT,
                             "ms_per_batch": statistics.mean(whole_ms),
                             "ms_per_batch_median": statistics.median(whole_ms),
                             "note": "one batch at a time, hops + incremental gather (the shipped graph)",
                             "hops_then_full_gather_ms": 1e3 * dev_s_single / args.steps},
            "roofline": {"kernel": "wg::gather_kernel", "bound": bound, "achieved": achieved, "peak": peak_used,
                         "unit": "GB/s", "frac": achieved / peak_used,
                         "traffic": gather_traffic() if wd == 1 else None,
                         "peak_source": peak_src_used,
                         "algorithmic_bytes_per_launch": alg_bytes / args.steps,
                         "gather_ms_per_launch": 1e3 * gather_s / args.steps,
                         "gather_share_of_single_batch": gather_s / (sum(step_ms) / 1e3),
                         "timed_in": "pass A (one batch at a time, events on the launching stream)"},
            "cpu_baseline": cpu,
            "stages_ms": stages,
            "paper_context": PAPER_CONTEXT,
            "e2e": {"value": e2e_val, "unit": UNIT, "h2d_bytes_per_step": S * 8,
                    "d2h_bytes_per_step": e2e_d2h, "batches": len(todo),
                    "note": f"public API (MiniBatchLoader, {P} batches in flight): per batch pinned-host seeds "
                            "H2D + batch graph + per-hop counts D2H, host-timed from first submit to last "
                            "batch handed out"},
            # our kernels per batch: 4 per hop (sample, insert, flag-scan, relabel) + the gather (pass A)
            # or + one gather_rows per hop (the shipped incremental graph: passes A' and B)
            "gpu_launches": args.steps * (4 * len(p.fanouts) + 1) + args.steps * (1 + P) * 5 * len(p.fanouts),
            "clocks": clk,
            "wall_s_timed_region": wall,
            "workload_stats": {**wdesc, "edges_per_hop_mean": hc[:, :, 0].mean(0).tolist(),
                               "unique_per_hop_mean": hc[:, :, 1].mean(0).tolist(),
                               "unique_bound_per_hop": pipes[0].U_cap, "rows_gathered_mean": float(rows.mean()),
                               "row_bytes": rb},
            "setup": {"total_s": setup_s, **info},
        }
        emit(line, args)
    torch.cuda.synchronize()
    for h in handles[1:]:
        h.destroy()
    dsm.destroy()
    if world > 1:
        dist.destroy_process_group()
    return line


def gather_traffic():
    """dram read+write bytes per launch of the gather kernel from the committed
    `ncu --set full` summary (profiles/latest_gather_ncu.json), or None."""
    pth = os.path.join(ROOT, "profiles", "latest_gather_ncu.json")
    if not os.path.exists(pth):
        return None
    with open(pth) as f:
        d = json.load(f)
    return d.get("dram_bytes_per_launch")


def bench_sweep(args):
    """Config 4 (BASELINE.json configs[3]): feature-gather sweep over row sizes on a
    100M-row table (the paper's Fig. 8 random-segment experiment, L240/L266): 1M
    uniform random ids per rank, dims 64..1024 x fp16/fp32.  Cells whose table does not
    fit one GPU are reported as skipped (they need W >= 2)."""
    import torch

    import paper_conf_sc_yanglql22_b200 as pkg
    from synth import features as sfeat
    from synth import gpu as sgpu
    from synth import presets, seeds
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    n = args.sweep_rows
    R = args.sweep_ids
    peak, peak_src = peaks()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    ids = torch.from_numpy(seeds.gather_ids(n, R, presets.SEED_BASE, 0)).to(dev)
    cells = []
    grid = [("fp16", d) for d in (2, 4, 8, 16, 32)]  # 4-64 B segments (Fig. 8's small sizes, NEXT #3)
    grid += [(t, d) for t in ("fp16", "fp32") for d in (64, 128, 256, 512, 768, 1024)]
    if args.sweep_cells:
        grid = [(c.split(":")[0], int(c.split(":")[1])) for c in args.sweep_cells.split(",")]
    else:
        # every cell in a fresh process: after the 100+ GB tables of the large cells the allocator's
        # physical memory is fragmented and a later table can land on small pages (measured: a 256 B
        # cell at 0.58 after the 1.5 KB cell in the same process, 0.85 in a fresh one)
        for dtype, dim in grid:
            r = subprocess.run([sys.executable, os.path.abspath(__file__), "--sweep", "--sweep-cells", f"{dtype}:{dim}",
                                "--steps", str(args.steps), "--sweep-rows", str(n), "--sweep-ids", str(R)],
                               capture_output=True, text=True, timeout=900)
            lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
            if r.returncode != 0 or not lines:
                cells.append({"dtype": dtype, "dim": dim, "error": (r.stderr or r.stdout)[-300:]})
                continue
            cells += json.loads(lines[-1])["cells"]
        grid = []
    for dtype, dim in grid:
        if True:
            rb = dim * sfeat.elt_bytes(dtype)
            pitch = (rb + 63) // 64 * 64
            need = n * pitch + n * 8 + R * rb
            free, _ = torch.cuda.mem_get_info()
            if need > 0.9 * free:
                cells.append({"dtype": dtype, "dim": dim, "row_bytes": rb, "skipped": f"table {n * pitch / 1e9:.0f} GB "
                              "does not fit one GPU (needs W >= 2)"})
                continue
            dsm = pkg.DSM(n, 0, dim, dtype, 1, device=0)
            sgpu.fill_dsm_features_gpu(dsm, presets.FEAT_SEED, 0, 1, dim, sfeat.WG_DTYPE_CODE[dtype])
            out = torch.empty((R, rb), dtype=torch.uint8, device=dev)
            for _ in range(3):
                dsm.gather(ids, out=out)
            torch.cuda.synchronize()
            ts = []
            for i in range(args.steps):
                flush.fill_(i & 0xFF)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                dsm.gather(ids, out=out)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1) / 1e3)
            assert dsm.device_error() == 0
            t = statistics.median(ts)
            algo = R * rb / t / 1e9
            cells.append({"dtype": dtype, "dim": dim, "row_bytes": rb, "ms": t * 1e3, "algo_gbs": algo,
                          "hbm_gbs_read_plus_write": 2 * algo, "frac_of_hbm_roofline": 2 * algo / peak})
            del out
            dsm.destroy()
            torch.cuda.empty_cache()
    measured = [c for c in cells if "ms" in c]
    best = max(measured, key=lambda c: c["frac_of_hbm_roofline"]) if measured else \
        {"hbm_gbs_read_plus_write": None, "frac_of_hbm_roofline": None}
    line = {"metric": "feature gather GB/s vs HBM roofline (config 4 sweep, W=1)", "value": best["hbm_gbs_read_plus_write"],
            "unit": "GB/s", "n_gpus": 1, "steps": args.steps, "warmup": 3, "higher_is_better": True,
            "config": {"workload": "gather-sweep", "rows": n, "ids_per_rank": R, "ids": "uniform with replacement",
                       "l2": "flushed between gathers"},
            "roofline": {"bound": "hbm", "peak": peak, "unit": "GB/s", "peak_source": peak_src,
                         "frac": best["frac_of_hbm_roofline"]},
            "cells": cells}
    emit(line, args)


def bench_latency(args):
    """NEXT #3 / PAPER.md Table I (L66-80): dependent 8 B load latency vs span (8..128 GB) of a
    DSM shard, one thread, `accesses` chained loads.  W=1: local HBM (the P2P column needs W>1)."""
    import torch

    import paper_conf_sc_yanglql22_b200 as pkg
    torch.cuda.set_device(0)
    free, _ = torch.cuda.mem_get_info()
    gib = 1 << 30
    spans = [s * gib for s in (1, 8, 16, 32, 64, 128) if s * gib < 0.85 * free]
    rows = max(spans) // 512
    dsm = pkg.DSM(rows, 0, 128, "fp32", 1, device=0)   # 512 B rows, filled with generator bits
    from synth import gpu as sgpu
    from synth import presets
    sgpu.fill_dsm_features_gpu(dsm, presets.FEAT_SEED, 0, 1, 128, 0)
    torch.cuda.synchronize()
    res = []
    for sp in spans:
        dsm.chase(0, sp, 2000)                            # warm-up (TLB, clocks)
        ns = statistics.median(dsm.chase(0, sp, args.chase_accesses) for _ in range(3))
        res.append({"span_gb": sp / gib, "ns_per_access": ns})
    dsm.destroy()
    line = {"metric": "dependent-load latency through a DSM shard (Table I analogue, local HBM, W=1)",
            "value": res[-1]["ns_per_access"], "unit": "ns", "higher_is_better": False,
            "config": {"accesses": args.chase_accesses, "threads": 1, "paper_A100_p2p_us": [1.35, 1.37, 1.43, 1.51, 1.56],
                       "paper_A100_um_us": [20.8, 29.6, 32.5, 35.3, 35.8]},
            "spans": res}
    emit(line, args)


def bench_layer(args):
    """NEXT #2 measurement: g-SpMM mean aggregation (GraphSAGE layer input) on a prepared
    products-shaped batch -- the last hop's CSR and the gathered features."""
    import torch

    import paper_conf_sc_yanglql22_b200 as pkg
    from paper_conf_sc_yanglql22_b200 import layers, loader
    from synth import presets, seeds
    torch.cuda.set_device(0)
    p = presets.get(args.config)
    dsm, _ = loader.build_dsm(p)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_dup=True)
    S = torch.from_numpy(seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, 5)).cuda()
    pipe.run(S, seeds.rng_seed(presets.RNG_BASE, 5))
    torch.cuda.synchronize()
    last, prev = pipe.hops[-1], pipe.hops[-2]
    T = int(prev["num_unique"].item())
    E = int(last["num_edges"].item())
    U = int(last["num_unique"].item())
    D = p.feat_dim
    X = pipe.X_rows[:U].contiguous().view(torch.float32).reshape(U, D) if p.feat_dtype == "fp32" \
        else torch.rand(U, D, device="cuda")
    row_ptr, sub_col, dup = last["row_ptr"][:T + 1], last["sub_col"][:E], last["dup"][:U]
    dY = torch.rand(T, D, device="cuda")
    peak, peak_src = peaks()
    res = {}
    for name, fn, alg in (
            ("forward", lambda: layers.spmm_mean_forward(row_ptr, sub_col, X), (E + T) * D * 4 + E * 4 + T * 8),
            ("backward", lambda: layers.spmm_mean_backward(row_ptr, sub_col, dup, dY, U),
             (T + E) * D * 4 + U * D * 4 + E * 4 + T * 8)):
        for _ in range(3):
            fn()
        ts = []
        for _ in range(args.steps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        t = statistics.median(ts)
        res[name] = {"ms": t * 1e3, "algorithmic_bytes": alg, "achieved_gbs": alg / t / 1e9,
                     "frac_of_hbm_roofline": alg / t / 1e9 / peak}
    dsm.destroy()
    line = {"metric": "g-SpMM mean aggregation on the prepared batch (NEXT #2)", "value": res["forward"]["achieved_gbs"],
            "unit": "GB/s", "higher_is_better": True, "n_gpus": 1, "steps": args.steps,
            "config": {"workload": p.name, "rows": T, "edges": E, "x_rows": U, "dim": D, "dtype": "fp32"},
            "roofline": {"bound": "hbm", "peak": peak, "peak_source": peak_src}, "results": res}
    emit(line, args)


def bench_compare_gather(args):
    """NEXT #1 / PAPER.md Fig. 10 (L297-305): the P2P global gather (one kernel, L182) vs the
    distributed-memory five-step gather (bucket, all-to-all ids, local gather, all-to-all rows,
    reorder, L178-180) on the same ids.  Under torchrun (W>1) the all-to-alls run on NCCL; at
    W=1 they are local copies, so the ratio shows the extra memory passes only."""
    import torch
    import torch.distributed as dist

    import paper_conf_sc_yanglql22_b200 as pkg
    from paper_conf_sc_yanglql22_b200 import loader
    from paper_conf_sc_yanglql22_b200.nccl_gather import DistributedGather
    from synth import presets, seeds
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0")) % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    ag = None
    if world > 1:
        if torch.cuda.device_count() >= world:
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
        ag = pkg.TorchDistAllgather(device=dev)
    p = presets.get(args.config)
    dsm, _ = loader.build_dsm(p, rank=rank, world=world, device=local, allgather=ag)
    dg = DistributedGather(dsm)
    ids = torch.from_numpy(seeds.gather_ids(p.n, args.sweep_ids, presets.SEED_BASE, rank)).to(dev)
    out = torch.empty((ids.numel(), dsm.row_bytes), dtype=torch.uint8, device=dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    res = {}
    for name, fn in (("p2p_one_kernel", lambda: dsm.gather(ids, out=out)), ("distributed_five_step", lambda: dg.gather(ids, out=out))):
        for _ in range(3):
            fn()
        ts = []
        for i in range(args.steps):
            flush.fill_(i & 0xFF)
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        t = statistics.median(ts)
        if world > 1:
            tt = torch.tensor([t], dtype=torch.float64)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            t = float(tt.item())
        res[name] = {"ms": t * 1e3, "algo_gbs_per_gpu": ids.numel() * dsm.row_bytes / t / 1e9}
    assert dsm.device_error() == 0
    if rank == 0:
        line = {"metric": "global gather: P2P (DSM, one kernel) vs distributed-memory five-step (Fig. 10 analogue)",
                "value": res["distributed_five_step"]["ms"] / res["p2p_one_kernel"]["ms"], "unit": "x (time ratio)",
                "higher_is_better": True, "n_gpus": world, "steps": args.steps,
                "config": {"workload": p.name, "ids_per_rank": int(ids.numel()), "row_bytes": dsm.row_bytes,
                           "exchange": "NCCL" if world > 1 and torch.cuda.device_count() >= world else
                           ("gloo via host" if world > 1 else "local copy (W=1)")},
                "results": res}
        emit(line, args)
    torch.cuda.synchronize()
    dsm.destroy()
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    if args.compare_gather:
        bench_compare_gather(args)
    elif args.layer:
        bench_layer(args)
    elif args.latency:
        bench_latency(args)
    elif args.sweep:
        bench_sweep(args)
    elif args.impl == "reference":
        bench_reference(args)
    else:
        bench_wg(args)


if __name__ == "__main__":
    main()
