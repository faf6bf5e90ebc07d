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
    ap.add_argument("--steps", type=int, default=200)
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
    ap.add_argument("--placement", default="dsm", choices=["dsm", "csr-replicated", "replicas"],
                    help="dsm (default, the paper's method): graph + features row-sharded over the W GPUs, remote "
                         "rows read over NVLink; csr-replicated (SURVEY 8(e)(ii) lever, labelled): the whole CSR on "
                         "every GPU (local sampling), features row-sharded (the gather crosses NVLink); replicas "
                         "(labelled): every GPU holds the whole graph + table (a W=1 DSM each), no NVLink traffic")
    ap.add_argument("--north-star", default="papers100m",
                    help="also measure this workload (the one the >= 6x scaling target is stated on) at the same N "
                         "and put it under north_star_workload ('' to skip)")
    ap.add_argument("--north-star-steps", type=int, default=10)
    ap.add_argument("--no-parity", dest="parity", action="store_false",
                    help="skip the per-rank oracle check of two batches after the timed passes")
    ap.add_argument("--chase-accesses", type=int, default=100_000)
    ap.add_argument("--latency-spans", default="1,8,16,32,64,128", help="--latency: spans in GiB (comma list)")
    ap.add_argument("--col64", action="store_true",
                    help="store col_idx as int64 (default: uint32, WG_DSM_COL32, whenever the node ids fit)")
    ap.add_argument("--hashed", action="store_true",
                    help="Append Unique in a hash table even when the direct table fits (WG_DSM_HASHED)")
    ap.add_argument("--x-pitch", type=int, default=None,
                    help="diagnostics: output row pitch of X (default: DSM.out_pitch(), the row rounded up to 32 B)")
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
def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or None


def run_oracle(preset, batches, sample_s, rank=0, world=1):
    """Time the CPU oracle (as it stands, single-threaded, pinned to one host core) on whole batches of
    the same workload; returns (seeds/s, seconds of oracle work, batches done, cores used, host info)."""
    import contextlib

    import oracle
    from synth import presets, providers, seeds
    before = sorted(os.sched_getaffinity(0))
    host = {"cpu_model": cpu_model(), "cores_available_before_pinning": len(before), "os_cpu_count": os.cpu_count()}
    os.sched_setaffinity(0, {before[0]})
    rows = providers.host_row_provider(preset.graph())
    feats = providers.host_feat_provider(preset)
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
    cores = len(os.sched_getaffinity(0))
    os.sched_setaffinity(0, set(before))
    return done * preset.seeds_per_batch / spent[0], spent[0], done, cores, host


def bench_reference(args):
    from synth import presets
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    p = presets.get(args.config)
    per_step = []
    total_s = 0.0
    for k in range(args.warmup + args.steps):
        v, s, done, cores, host = run_oracle(p, [k], 0.0)
        if k >= args.warmup:
            per_step.append(s)
            total_s += s
    value = args.steps * p.seeds_per_batch / total_s
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total_s / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64+fp32-bytes",
            "data": "synthetic", "config": workload_config(p, 1),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", **host,
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
    par = {"dsm": f"dsm-w{W} (row-sharded CSR+features, P2P loads, no hot-path collective)",
           "csr-replicated": f"csr-replicated-w{W} (SURVEY 8(e)(ii) lever: whole CSR on every GPU, features "
                             "row-sharded, gather P2P over NVLink, no hot-path collective)",
           "replicas": f"replicas-x{W} (SURVEY 8(e) lever: whole graph + table on every GPU, no NVLink, no "
                       "hot-path collective)"}[placement]
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

def measure_ceilings(dsm, reps=3):
    """The ceilings the latency-bound prep kernels are measured against, on this box:
    independent random 8 B / 32 B loads over the col_idx shard (the sampler's S1-S2 accesses) and over
    an L2-sized span (the flag scan's table reads), and independent 64-bit L2 atomics (probe CAS, claim
    CAS, atomicMin) on a 2^21-word (17 MB) table, the size of a products hop-2 hash table (S3)."""
    import ctypes

    import torch

    from paper_conf_sc_yanglql22_b200._lib import check, lib
    dev = dsm.device
    sink = torch.zeros(1, dtype=torch.int64, device=dev)
    st = torch.cuda.current_stream(dev)
    _, col, _ = dsm.local_view()
    small = torch.zeros(16 << 20, dtype=torch.uint8, device=dev)
    table = torch.zeros(1 << 21, dtype=torch.int64, device=dev)
    n = ctypes.c_int64()

    def timed(fn):
        best = None
        for _ in range(reps + 1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            fn()
            e1.record(st)
            e1.synchronize()
            t = e0.elapsed_time(e1) / 1e3
            best = t if best is None else min(best, t)
        return n.value / best

    out = {}
    col_bytes = col.numel() * col.element_size()   # 4 B entries with WG_DSM_COL32
    for name, buf, span, width in (("random_8B_loads_per_s_col_shard", col, col_bytes, 8),
                                   ("random_32B_loads_per_s_col_shard", col, col_bytes, 32),
                                   ("random_8B_loads_per_s_16MB", small, small.numel(), 8)):
        out[name] = timed(lambda: check(lib().wg_micro_random_read(ctypes.c_void_p(buf.data_ptr()), span, width, 16, 8,
                                                                    ctypes.c_void_p(sink.data_ptr()), ctypes.byref(n),
                                                                    ctypes.c_void_p(st.cuda_stream))))
    for name, op in (("l2_cas_probe_per_s_17MB", 0), ("l2_cas_claim_per_s_17MB", 1), ("l2_atomic_min_per_s_17MB", 2)):
        out[name] = timed(lambda: check(lib().wg_micro_atomics(ctypes.c_void_p(table.data_ptr()), table.numel(), op, 16, 8,
                                                                ctypes.c_void_p(sink.data_ptr()), ctypes.byref(n),
                                                                ctypes.c_void_p(st.cuda_stream))))
    out["col_shard_bytes"] = col_bytes
    out["note"] = ("wg_micro_random_read / wg_micro_atomics: 148 SMs x 8 blocks x 256 threads, 8 independent "
                   "operations in flight per thread, best of 3")
    return out


def hop_kernels(m, direct=False):
    """Kernel stages of one wg_sample_hop (the stage events the library records); with the direct key
    table (direct=True) the sampler inserts every key and there is no insert pass."""
    return ("sample", "flag", "relabel") if direct else ("sample", "insert", "flag", "relabel")


def stage_breakdown(pipe, seeds_dev, rngs, flush, ceil=None, nb=20):
    """SURVEY 8(d) per-kernel device times of one batch (outside every timed region): each hop's sampler,
    insert, flag scan and relabel (wg_dsm_set_stage_events: an event after every kernel, eager launches,
    everything on one stream), then the whole gather; L2 flushed before each batch; medians.  With the
    measured ceilings every prep kernel gets a fraction of its own bound: per hop with T targets and E
    sampled edges, the sampler's T + E random loads (row_ptr pairs, col entries) against the random 8 B
    load rate over the col shard, the insert's T + E keys against the L2 probe-CAS rate, the flag scan's
    and the relabel's E random reads against the random 8 B load rate over an L2-sized span."""
    import torch
    st = torch.cuda.current_stream()
    H = len(pipe.fanouts)
    direct = not pipe.dsm.hop_insert_pass()   # the sampler inserts: no insert kernel

    def hop_kernels_(m):
        return hop_kernels(m, direct)
    acc = {f"hop{h}_{k}": [] for h in range(H) for k in hop_kernels_(pipe.fanouts[h])}
    acc["gather"] = []
    cnt = []
    for b in range(nb + 2):
        pipe.set_inputs(seeds_dev[b % len(seeds_dev)], rngs[b % len(rngs)])
        if flush is not None:
            flush.fill_(b & 0xFF)
        evs = [[torch.cuda.Event(enable_timing=True) for _ in range(len(hop_kernels_(m)) + 1)] for m in pipe.fanouts]
        for row in evs:               # create the events (torch creates them lazily at the first record)
            for e in row:
                e.record(st)
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        tgt, tcap, tn = pipe.seeds, pipe.max_seeds, pipe.n_seeds
        for h, m in enumerate(pipe.fanouts):
            bb = pipe.hops[h]
            evs[h][0].record(st)
            pipe.dsm.set_stage_events(evs[h][1:])
            pipe.dsm.sample_hop(tgt, m, 0, h, n_targets_dev=tn, seed_dev=pipe.rng_seed, out=bb, cap=tcap, stream=st)
            pipe.dsm.set_stage_events([])
            tgt, tcap, tn = bb["unique"], pipe.U_cap[h], bb["num_unique"]
        g0.record(st)
        pipe.enqueue_gather(st)
        g1.record(st)
        torch.cuda.synchronize()
        if b >= 2:
            for h, m in enumerate(pipe.fanouts):
                for k, kind in enumerate(hop_kernels_(m)):
                    acc[f"hop{h}_{kind}"].append(evs[h][k].elapsed_time(evs[h][k + 1]))
            acc["gather"].append(g0.elapsed_time(g1))
            cnt.append(pipe.counts_dev.cpu().numpy().copy())
    out = {n: statistics.median(v) for n, v in acc.items()}
    for h, m in enumerate(pipe.fanouts):
        out[f"hop{h}"] = sum(out[f"hop{h}_{k}"] for k in hop_kernels_(m))
    c = np.mean(cnt, axis=0)
    fr = {}
    if ceil:
        T = float(pipe.max_seeds)
        for h, m in enumerate(pipe.fanouts):
            E, U = float(c[h, 0]), float(c[h, 1])
            t = {k: out[f"hop{h}_{k}"] / 1e3 for k in hop_kernels_(m)}
            phases = {"random_loads": (T + E) / ceil["random_8B_loads_per_s_col_shard"],
                      "l2_probe_cas": (T + E) / ceil["l2_cas_probe_per_s_17MB"],
                      "l2_reads": E / ceil["random_8B_loads_per_s_16MB"]}
            d = {"targets": T, "edges": E, "unique": U}
            d["sample"] = phases["random_loads"] / t["sample"]
            if "insert" in t:
                d["insert"] = phases["l2_probe_cas"] / t["insert"]
            d["flag"] = phases["l2_reads"] / t["flag"]
            d["relabel"] = E / t["relabel"] / ceil["random_8B_loads_per_s_16MB"]
            fr[f"hop{h}"] = d
            T = U
        kinds = ("sample", "insert", "flag", "relabel")
        worst = min(((h, k, v) for h, d in fr.items() for k, v in d.items() if k in kinds), key=lambda x: x[2])
        fr["furthest_below"] = {"hop": worst[0], "kernel": worst[1], "frac": worst[2]}
    out["frac"] = fr
    out["unique_format"] = ["wide", "compact", "direct"][pipe.dsm.unique_format()]
    out["note"] = ("median ms per kernel of one batch (eager launches, an event after every kernel, L2 flushed per "
                   "batch; hop h = wg_sample_hop); frac = each kernel's operation rate over its measured ceiling "
                   "(ceilings)")
    return out


def emit(line, args):
    s = json.dumps(line)
    print(s, flush=True)
    if args.out:
        with open(args.out, "a") as f:
            f.write(s + "\n")


# ----------------------------------------------------------------------------- GPU arm
class Dist:
    """Process placement: one rank per GPU (rank r on cuda:(LOCAL_RANK % device_count)); NCCL for the
    setup-time plumbing (handle allgather, barriers, max over ranks) when every rank has its own GPU,
    gloo when ranks share one (a test box with fewer GPUs than ranks).  Never on the hot path."""

    def __init__(self):
        import torch
        import torch.distributed as dist

        import paper_conf_sc_yanglql22_b200 as pkg
        self.dist = dist
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        local = int(os.environ.get("LOCAL_RANK", "0"))
        self.ndev = torch.cuda.device_count()
        self.local = local % self.ndev
        torch.cuda.set_device(self.local)
        self.dev = torch.device("cuda", self.local)
        self.ag, self.backend = None, None
        local_world = int(os.environ.get("LOCAL_WORLD_SIZE", self.world))
        self.shared_gpu = self.world > 1 and self.ndev < local_world   # "remote" rows are then local HBM
        if self.world > 1:
            self.backend = "gloo" if self.shared_gpu else "nccl"
            if self.backend == "nccl":
                dist.init_process_group("nccl", device_id=self.dev)
            else:
                dist.init_process_group("gloo")
            self.ag = pkg.TorchDistAllgather(device=self.dev)

    def barrier(self):
        if self.world > 1:
            self.dist.barrier()

    def max(self, x):
        import torch
        if self.world == 1:
            return x
        t = torch.tensor([float(x)], dtype=torch.float64, device=self.dev if self.backend == "nccl" else "cpu")
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX)
        return float(t.item())

    def all_true(self, ok):
        return self.max(0.0 if ok else 1.0) == 0.0

    def close(self):
        if self.world > 1:
            self.dist.destroy_process_group()


PLACEMENTS = ("dsm", "csr-replicated", "replicas")


class Workload:
    """One preset on this rank: the DSM (per --placement), P batch pipelines on P workspace forks and
    P streams, the rank's batches (b = k * W + r), and the graphs bench.py replays."""

    def __init__(self, args, p, d, P, placement, n_single, n_conc):
        import torch

        import paper_conf_sc_yanglql22_b200 as pkg
        from paper_conf_sc_yanglql22_b200 import loader
        from paper_conf_sc_yanglql22_b200 import pipeline as pipemod
        from synth import presets, seeds
        self.p, self.d, self.P, self.placement = p, d, P, placement
        S = p.seeds_per_batch
        t0 = time.perf_counter()
        col32 = False if args.col64 else None   # None: the loader's default (uint32 when the ids fit)
        hashed = pkg.WG_DSM_HASHED if args.hashed else 0
        if placement == "replicas":   # every rank its own whole copy (a W=1 DSM); batches still b = r mod W
            self.dsm, self.info = loader.build_dsm(p, rank=0, world=1, device=d.local, allgather=None, col32=col32,
                                                   flags=hashed)
        else:
            flags = (pkg.WG_DSM_CSR_REPLICATED if placement == "csr-replicated" else 0) | hashed
            self.dsm, self.info = loader.build_dsm(p, rank=d.rank, world=d.world, device=d.local, allgather=d.ag,
                                                   flags=flags, col32=col32)
        self.info["col_idx_bytes"] = 4 if self.dsm.flags & pkg.WG_DSM_COL32 else 8
        self.setup_s = time.perf_counter() - t0
        # the W of the feature table (NVLink share (W-1)/W of the gathered rows)
        self.w_feat = 1 if placement == "replicas" else d.world
        self.handles = [self.dsm] + [self.dsm.fork() for _ in range(P - 1)]
        self.pipes = [pkg.MiniBatchPipeline(h, p.fanouts, S, x_pitch=args.x_pitch) for h in self.handles]
        self.streams = [torch.cuda.Stream(device=d.dev) for _ in range(P)]
        self.n_single = n_single
        self.batches = [k * d.world + d.rank for k in range(n_single + n_conc)]
        self.seeds_dev = [torch.from_numpy(seeds.seed_nodes(p.n, S, presets.SEED_BASE, b)).to(d.dev)
                          for b in self.batches]
        self.rngs = [seeds.rng_seed(presets.RNG_BASE, b) for b in self.batches]
        # each batch's inputs resident in HBM as the pipeline's packed input layout: one D2D copy per batch
        self.packed_dev = [pipemod.pack_inputs(s_, r_, d.dev) for s_, r_ in zip(self.seeds_dev, self.rngs)]
        self.flush = None if args.no_flush else torch.empty(512 << 20, dtype=torch.uint8, device=d.dev)
        occ_b = args.gather_occupancy
        if occ_b is None:
            occ_b = pipemod.THROUGHPUT_GATHER_OCCUPANCY if P >= 4 else 0
        self.occ_b = occ_b
        for k in range(args.warmup):              # warm-up (eager)
            for pl in self.pipes:
                pl.run(self.seeds_dev[k], self.rngs[k])
        torch.cuda.synchronize()
        # per pipeline: hops only | whole gather (the roofline kernel) | the batch as shipped (incremental
        # gather) | the same with the throughput gather occupancy
        self.graphs = []
        for pl, st in zip(self.pipes, self.streams):
            if args.no_graph:
                self.graphs.append(None)
                continue
            st.wait_stream(torch.cuda.current_stream())
            g = {k: torch.cuda.CUDAGraph() for k in ("prep", "gather", "whole", "tput")}
            with torch.cuda.graph(g["prep"], stream=st):
                pl.enqueue(gather=False)
            with torch.cuda.graph(g["gather"], stream=st):
                pl.enqueue_gather()
            with torch.cuda.graph(g["whole"], stream=st):
                pl.enqueue(gather=True, gather_occupancy=0)
            with torch.cuda.graph(g["tput"], stream=st):
                pl.enqueue(gather=True, gather_occupancy=occ_b)
            self.graphs.append(g)
        torch.cuda.synchronize()
        for k in range(args.warmup):              # warm the graphs
            for j in range(P):
                self.launch(j, k, "prep", self.streams[j])
                self.launch(j, None, "gather", self.streams[j])
                self.launch(j, k, "whole", self.streams[j])
                self.launch(j, k, "tput", self.streams[j])
        torch.cuda.synchronize()
        self.check_errors("warm-up")

    def launch(self, j, k, kind, st):
        """Batch k (None: keep the inputs) through pipeline j on stream st (inputs resident in HBM)."""
        import torch
        pl, g = self.pipes[j], self.graphs[j]
        with torch.cuda.stream(st):
            if k is not None:
                pl.set_inputs_packed(self.packed_dev[k])
            if g is not None:
                g[kind].replay()
            elif kind == "prep":
                pl.enqueue(gather=False)
            elif kind == "gather":
                pl.enqueue_gather()
            else:
                pl.enqueue(gather_occupancy=self.occ_b if kind == "tput" else 0)
        return pl

    def check_errors(self, where):
        for h in self.handles:
            err = h.device_error()
            assert err == 0, f"device error {err:#x} ({where})"

    def pass_a(self, steps, warmup):
        """One batch at a time: hops then the whole gather (the roofline kernel, events on its launching
        stream), then the batch as shipped (hops + incremental gather) for the single-batch latency."""
        import torch
        main = torch.cuda.current_stream()
        ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(steps)]
        rows = torch.zeros(steps, dtype=torch.int64, device=self.d.dev)
        counts = torch.zeros((steps, len(self.p.fanouts), 2), dtype=torch.int64, device=self.d.dev)
        for i in range(steps):
            k = warmup + i
            if self.flush is not None:
                self.flush.fill_(i & 0xFF)
            ev[i][0].record(main)
            pl = self.launch(0, k, "prep", main)
            ev[i][1].record(main)
            self.launch(0, None, "gather", main)
            ev[i][2].record(main)
            rows[i:i + 1].copy_(pl.hops[-1]["num_unique"])
            counts[i].copy_(pl.counts_dev)
        torch.cuda.synchronize()
        step_ms = [ev[i][0].elapsed_time(ev[i][2]) for i in range(steps)]
        gather_ms = [ev[i][1].elapsed_time(ev[i][2]) for i in range(steps)]
        evw = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(steps)]
        for i in range(steps):
            if self.flush is not None:
                self.flush.fill_(i & 0xFF)
            evw[i][0].record(main)
            self.launch(0, warmup + i, "whole", main)
            evw[i][1].record(main)
        torch.cuda.synchronize()
        whole_ms = [evw[i][0].elapsed_time(evw[i][1]) for i in range(steps)]
        return step_ms, gather_ms, whole_ms, rows.cpu().numpy(), counts.cpu().numpy()

    def pass_b(self, steps, warmup, mode="both"):
        """The throughput number: P pipelines run continuously on P streams (pipeline j prepares batches
        j, j+P, ...), K steps of P batches timed as one region (events on the main stream, barrier +
        synchronize on both sides).  No L2 flush inside: the inputs (graph + table) are far larger than
        the 126 MB L2 and every batch is new."""
        import torch
        main = torch.cuda.current_stream()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        self.d.barrier()
        torch.cuda.synchronize()
        e0.record(main)
        for j in range(self.P):
            self.streams[j].wait_stream(main)
        for i in range(steps):
            for j in range(self.P):
                k = self.n_single + warmup + i * self.P + j
                if mode == "both":
                    self.launch(j, k, "tput", self.streams[j])
                    continue
                if mode != "gather":
                    self.launch(j, k, "prep", self.streams[j])
                if mode != "prep":
                    self.launch(j, None, "gather", self.streams[j])
        for j in range(self.P):
            main.wait_stream(self.streams[j])
        e1.record(main)
        torch.cuda.synchronize()
        self.d.barrier()
        return e0.elapsed_time(e1)

    def parity(self, ks):
        """Outside every timed region: batches ks (indices into this rank's batch list, e.g. ones the
        timed passes ran) through the shipped graph again, every hop array and the gathered bytes compared
        element by element with the CPU oracle (tolerance 0).  Returns the parity record, with the share
        of gathered rows owned by another rank (read over NVLink when every rank has its own GPU)."""
        import torch

        import oracle
        from synth import providers
        rows = providers.host_row_provider(self.p.graph())
        feats = providers.host_feat_provider(self.p)
        ok, checked, remote, total, t0 = True, [], 0, 0, time.perf_counter()
        pl = self.pipes[0]
        for k in ks:
            self.launch(0, k, "whole", torch.cuda.current_stream())
            torch.cuda.synchronize()
            S = self.seeds_dev[k].cpu().numpy()
            ref = oracle.minibatch(rows, feats, S, self.p.fanouts, self.rngs[k])
            for h in range(len(self.p.fanouts)):
                got, exp = pl.result(h), ref["hops"][h]
                for key in ("row_ptr", "nbrs", "unique", "sub_col"):
                    ok = ok and np.array_equal(got[key], exp[key])
            ok = ok and np.array_equal(pl.features(), ref["X"])
            U = ref["hops"][-1]["unique"]
            remote += int((U % self.w_feat != (self.d.rank % self.w_feat)).sum())
            total += len(U)
            checked.append(int(self.batches[k]))
        self.check_errors("parity")
        return {"batches": len(ks), "global_batch_ids": checked, "ok": bool(ok),
                "compared": "every hop's row_ptr, nbrs, unique, sub_col and the gathered feature bytes, "
                            "element by element against the CPU oracle (tolerance 0)",
                "remote_row_share": remote / max(total, 1), "oracle_s": time.perf_counter() - t0}

    def roofline(self, rows, gather_ms, steps):
        """Gather roofline: t_roof = max(2RB / HBM, (W-1)/W * RB / NVLink).  At W=1 (or
        replicas) every byte is local HBM (read + write); at W>1 with one GPU per rank the (W-1)/W remote
        share crosses NVLink and bounds the kernel."""
        peak, peak_src = peaks()
        rb = self.dsm.row_bytes
        R = float(rows.sum())
        hbm_bytes = 2 * R * rb
        wd = self.w_feat
        nvl_bytes = (wd - 1) / wd * R * rb
        gather_s = sum(gather_ms) / 1e3
        if nvl_bytes / NVLINK_GBS > hbm_bytes / peak and not self.d.shared_gpu:
            bound, alg, pk, src = "nvlink", nvl_bytes, NVLINK_GBS, NVLINK_SRC
        else:
            bound, alg, pk, src = "hbm", hbm_bytes, peak, peak_src
        achieved = alg / gather_s / 1e9
        return {"kernel": "wg::gather_kernel", "bound": bound, "achieved": achieved, "peak": pk, "unit": "GB/s",
                "frac": achieved / pk, "traffic": gather_traffic(self.p.name) if wd == 1 else None,
                "peak_source": src, "algorithmic_bytes_per_launch": alg / steps,
                "hbm_bytes_per_launch": hbm_bytes / steps, "nvlink_bytes_per_launch": nvl_bytes / steps,
                "nvlink_share_of_rows": (wd - 1) / wd, "gather_ms_per_launch": 1e3 * gather_s / steps,
                "timed_in": "pass A (one batch at a time, events on the launching stream)"}

    def destroy(self):
        import torch
        torch.cuda.synchronize()
        for h in self.handles[1:]:
            h.destroy()
        self.dsm.destroy()
        self.pipes, self.handles, self.graphs = [], [], []
        torch.cuda.empty_cache()


NVLINK_GBS = 770.0   # measured peer copy bandwidth per direction, B200_PROFILING.md (900 nominal)
NVLINK_SRC = "measured peer copy BW per direction (B200_PROFILING.md; 900 nominal)"


def whole_step_roofline(p, counts, rows, rb, ms_per_batch, w_feat):
    """Whole-step efficiency: SURVEY 8(d) algorithmic bytes of one batch (every hop's S1-S4 bytes + the
    gather's 2RB) / measured per-batch time / the HBM peak.  Per hop with T targets, E sampled edges and
    U unique: S1-S2 16 B row_ptr pair + 8 B row_ptr write per target, 8 B col read + 8 B id write per
    edge; S3-S4 8 B key read + 4 B sub_col write per edge + 8 B per unique id written."""
    peak, _ = peaks()
    T = p.seeds_per_batch
    prep = 0.0
    for h in range(len(p.fanouts)):
        E, U = counts[:, h, 0].mean(), counts[:, h, 1].mean()
        prep += 24 * T + 16 * E + 12 * E + 8 * U
        T = U
    R = rows.mean()
    gather = 2 * R * rb
    alg = prep + gather
    t = ms_per_batch / 1e3
    return {"algorithmic_bytes_per_batch": alg, "prep_bytes": prep, "gather_bytes": gather,
            "ms_per_batch": ms_per_batch, "achieved_gbs": alg / t / 1e9, "peak": peak, "frac": alg / t / 1e9 / peak,
            "floor_us_per_batch": alg / peak / 1e3,
            "note": "whole batch (all hops + gather) in the throughput pass vs its HBM floor; at W>1 the "
                    f"{(w_feat - 1)}/{w_feat} remote rows cross NVLink instead"}


def bench_wg(args):
    import torch

    import paper_conf_sc_yanglql22_b200 as pkg
    from synth import presets

    d = Dist()
    p = presets.get(args.config)
    S = p.seeds_per_batch
    P = max(1, args.concurrency)
    n_single = args.warmup + args.steps
    n_conc = args.warmup + args.steps * P
    wl = Workload(args, p, d, P, args.placement, n_single, n_conc)
    kph = 4 if wl.dsm.hop_insert_pass() else 3   # kernels per hop (wg_dsm_unique_format)
    clocks = ClockSampler(d.local)
    if d.rank == 0:
        clocks.start()
    d.barrier()
    torch.cuda.synchronize()
    wall0 = time.perf_counter()
    step_ms, gather_ms, whole_ms, rows, hc = wl.pass_a(args.steps, args.warmup)
    conc_ms = wl.pass_b(args.steps, args.warmup, args.pass_b)
    wall = time.perf_counter() - wall0
    clk = clocks.stop() if d.rank == 0 else None
    wl.check_errors("timed region")
    dev_s_single = d.max(sum(step_ms) / 1e3)
    dev_s_conc = d.max(conc_ms / 1e3)
    dev_s_whole = d.max(statistics.mean(whole_ms) / 1e3)
    value_conc = d.world * S * P * args.steps / dev_s_conc
    roof = wl.roofline(rows, gather_ms, args.steps)
    roof["gather_share_of_single_batch"] = sum(gather_ms) / sum(step_ms)
    # parity of this rank's batches against the oracle (outside the timed regions): the first batch of
    # pass A and the first of pass B (so N>1 runs carry a per-rank byte check, not only the error word)
    par = wl.parity([args.warmup, n_single + args.warmup]) if args.parity else None
    par_ok = d.all_true(par["ok"]) if par else None

    # e2e through the public API (MiniBatchLoader): every batch = H2D of its seeds from pinned host memory
    # + the batch graph + D2H of its per-hop counts, P batches in flight (as pass B), host-timed from the
    # first submit to the last batch handed out
    loader_ = pkg.MiniBatchLoader(wl.dsm, p.fanouts, S, depth=P, gather_occupancy=wl.occ_b)
    host_seeds = [wl.seeds_dev[k % n_single].cpu().pin_memory() for k in range(args.e2e_steps * P)]
    warm = [(host_seeds[k % len(host_seeds)], wl.rngs[k % n_single]) for k in range(2 * P)]
    for _ in loader_(warm):
        pass
    torch.cuda.synchronize()
    todo = [(host_seeds[k], wl.rngs[(n_single + k) % len(wl.rngs)]) for k in range(args.e2e_steps * P)]
    d.barrier()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in loader_(todo):
        pass
    e2e_s = time.perf_counter() - t
    assert loader_.device_error() == 0
    e2e_val = d.world * S * len(todo) / d.max(e2e_s)
    loader_.close()

    wdesc = workload_descriptors(wl.dsm, wl.pipes[0], wl.seeds_dev, wl.rngs) if d.rank == 0 else {}
    ceil = measure_ceilings(wl.dsm) if d.rank == 0 else None
    stages = stage_breakdown(wl.pipes[0], wl.seeds_dev, wl.rngs, wl.flush, ceil) if d.rank == 0 else {}
    whole_step = whole_step_roofline(p, hc, rows, wl.dsm.row_bytes, 1e3 * dev_s_conc / (args.steps * P), wl.w_feat)
    rb, info, setup_s, occ_b = wl.dsm.row_bytes, wl.info, wl.setup_s, wl.occ_b
    wl.destroy()
    del wl

    # the north-star workload (papers100M-shaped, the one the >= 6x scaling target is stated on) at the
    # same N, measured after the headline workload is torn down
    north = None
    if args.north_star and args.config != args.north_star:
        north = bench_north_star(args, d, presets.get(args.north_star), P)

    line = None
    if d.rank == 0:
        cpu = None
        if d.world == 1 and args.cpu_sample_s > 0:
            v, s_spent, done, cores, host = run_oracle(p, range(10_000, 10_100), args.cpu_sample_s)
            cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", **host,
                   "sample": f"{done} whole batches of {S} seeds (fanout {p.fanouts} + gather) of the same workload, "
                             f"{s_spent:.1f} s of single-threaded oracle work (row regeneration untimed)"}
        cfg = workload_config(p, d.world, wl_flush(args), args.placement)
        cfg["concurrent_batches_per_gpu"] = P
        cfg["gather_blocks_per_sm_throughput_pass"] = occ_b or "occupancy max"
        cfg["gpus_visible"] = d.ndev
        cfg["l2"] = ("pass A (single batch, roofline): L2 flushed between batches; pass B (value): continuous, "
                     "inputs (graph + features) >> 126 MB L2, every batch new")
        line = {
            "metric": METRIC, "value": value_conc, "unit": UNIT, "n_gpus": d.world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * dev_s_conc / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64 ids + fp32 feature bytes",
            "data": "synthetic (seeded power-law graph + procedural features, see DESIGN.md)",
            "config": cfg,
            "parity": None if par is None else {**par, "ok": par_ok, "ranks": d.world},
            "single_batch": {"value": d.world * S / dev_s_whole, "unit": UNIT,
                             "ms_per_batch": statistics.mean(whole_ms),
                             "ms_per_batch_median": statistics.median(whole_ms),
                             "note": "one batch at a time, hops + incremental gather (the shipped graph)",
                             "hops_then_full_gather_ms": 1e3 * dev_s_single / args.steps},
            "roofline": roof,
            "whole_step_roofline": whole_step,
            "cpu_baseline": cpu,
            "stages_ms": stages,
            "ceilings": ceil,
            "north_star_workload": north,
            "paper_context": PAPER_CONTEXT,
            "e2e": {"value": e2e_val, "unit": UNIT, "h2d_bytes_per_step": S * 8 + 16,
                    "d2h_bytes_per_step": len(p.fanouts) * 2 * 8, "batches": len(todo),
                    "note": f"public API (MiniBatchLoader, {P} batches in flight): per batch pinned-host seeds "
                            "+ (n_seeds, rng_seed) H2D, batch graph, per-hop counts D2H, host-timed from first "
                            "submit to last batch handed out"},
            # our kernels per batch: 3 per hop (sample, flag-scan, relabel; + insert with a hashed key table)
            # + one gather (pass A) or one gather_rows per hop (the shipped incremental graph: passes A' and B)
            "gpu_launches": args.steps * (kph * len(p.fanouts) + 1) + args.steps * (1 + P) * (kph + 1) * len(p.fanouts),
            "clocks": clk,
            "wall_s_timed_region": wall,
            "workload_stats": {**wdesc, "edges_per_hop_mean": hc[:, :, 0].mean(0).tolist(),
                               "unique_per_hop_mean": hc[:, :, 1].mean(0).tolist(),
                               "rows_gathered_mean": float(rows.mean()), "row_bytes": rb},
            "setup": {"total_s": setup_s, **info},
        }
        emit(line, args)
    torch.cuda.synchronize()
    if par is not None and not par_ok:
        raise SystemExit("parity check against the oracle FAILED")
    d.close()
    return line


def wl_flush(args):
    return not args.no_flush


def bench_north_star(args, d, p, P):
    """The papers100M-shaped workload at the same N and placement: pass A (gather roofline), pass B (the
    throughput, as the headline) and the per-rank oracle parity of two batches."""
    import torch
    steps = max(3, min(args.steps, args.north_star_steps))
    n_single = args.warmup + steps
    wl = Workload(args, p, d, P, args.placement, n_single, args.warmup + steps * P)
    step_ms, gather_ms, whole_ms, rows, hc = wl.pass_a(steps, args.warmup)
    conc_ms = wl.pass_b(steps, args.warmup)
    wl.check_errors("north-star timed region")
    dev_s_conc = d.max(conc_ms / 1e3)
    dev_s_whole = d.max(statistics.mean(whole_ms) / 1e3)
    roof = wl.roofline(rows, gather_ms, steps)
    par = wl.parity([args.warmup, n_single + args.warmup]) if args.parity else None
    par_ok = d.all_true(par["ok"]) if par else None
    S = p.seeds_per_batch
    out = {"workload": p.name, "note": p.note, "value": d.world * S * P * steps / dev_s_conc, "unit": UNIT,
           "steps": steps, "ms_per_step": 1e3 * dev_s_conc / steps,
           "single_batch_ms": 1e3 * dev_s_whole, "roofline": roof,
           "whole_step_roofline": whole_step_roofline(p, hc, rows, wl.dsm.row_bytes, 1e3 * dev_s_conc / (steps * P),
                                                      wl.w_feat),
           "parity": None if par is None else {**par, "ok": par_ok, "ranks": d.world},
           "unique_per_hop_mean": hc[:, :, 1].mean(0).tolist(), "setup": {"total_s": wl.setup_s, **wl.info},
           "parallelism": workload_config(p, d.world, True, args.placement)["parallelism"]}
    wl.destroy()
    if par is not None and not par_ok:
        raise SystemExit("north-star parity check against the oracle FAILED")
    return out


def gather_traffic(workload):
    """dram read+write bytes per launch of the gather kernel on this workload, from the committed
    `ncu --set full` capture of the same build (profiles/latest_gather_ncu.json), or None."""
    pth = os.path.join(ROOT, "profiles", "latest_gather_ncu.json")
    if not os.path.exists(pth):
        return None
    with open(pth) as f:
        d = json.load(f)
    return d.get(workload, {}).get("dram_bytes_per_launch")


def bench_sweep(args):
    """Config 4 (BASELINE.json configs[3]): feature-gather sweep over row sizes on a 100M-row table
    (the paper's Fig. 8 random-segment experiment, L240/L266): 1M uniform random ids per rank, dims
    64..1024 x fp16/fp32 (+ the 4-64 B segments of NEXT #3).  Under torchrun the table is row-sharded over
    the W GPUs (o(v) = v mod W) and every rank gathers its own ids at once (barrier, max over ranks), so
    (W-1)/W of the rows cross NVLink: AlgoBW = R*B/t per GPU, BusBW = (W-1)/W * AlgoBW (A17), against
    t_roof = max(2RB / HBM, (W-1)/W * RB / NVLink).  Every cell byte-checks 4096 sampled rows against the
    closed-form generator.  Cells whose shard does not fit one GPU are reported as skipped."""
    import torch

    import paper_conf_sc_yanglql22_b200 as pkg
    from synth import features as sfeat
    from synth import gpu as sgpu
    from synth import presets, seeds
    d = Dist()
    n = args.sweep_rows
    R = args.sweep_ids
    W = d.world
    peak, peak_src = peaks()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=d.dev)
    ids_np = seeds.gather_ids(n, R, presets.SEED_BASE, d.rank)
    ids = torch.from_numpy(ids_np).to(d.dev)
    check_idx = np.random.default_rng(d.rank).choice(R, min(R, 4096), replace=False)
    cells = []
    grid = [("fp16", dd) for dd in (2, 4, 8, 16, 32)]  # 4-64 B segments (Fig. 8's small sizes, NEXT #3)
    grid += [(t, dd) for t in ("fp16", "fp32") for dd in (64, 128, 256, 512, 768, 1024)]
    if args.sweep_cells:
        grid = [(c.split(":")[0], int(c.split(":")[1])) for c in args.sweep_cells.split(",")]
    elif W == 1:
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
        rb = dim * sfeat.elt_bytes(dtype)
        pitch = (rb + 63) // 64 * 64
        n_local = (n + W - 1) // W
        need = n_local * pitch + R * rb
        free, _ = torch.cuda.mem_get_info()
        fits = d.all_true(need < 0.9 * free)
        if not fits:
            cells.append({"dtype": dtype, "dim": dim, "row_bytes": rb, "skipped": f"shard {n_local * pitch / 1e9:.0f} GB "
                          f"does not fit one GPU at W={W}"})
            continue
        dsm = pkg.DSM(n, 0, dim, dtype, 1, rank=d.rank, world_size=W, device=d.local, allgather=d.ag)
        sgpu.fill_dsm_features_gpu(dsm, presets.FEAT_SEED, d.rank, W, dim, sfeat.WG_DTYPE_CODE[dtype])
        torch.cuda.synchronize()
        d.barrier()                                           # every shard filled before anyone reads
        out = torch.empty((R, rb), dtype=torch.uint8, device=d.dev)
        for _ in range(3):
            dsm.gather(ids, out=out)
        torch.cuda.synchronize()
        ts = []
        for i in range(args.steps):
            flush.fill_(i & 0xFF)
            torch.cuda.synchronize()
            d.barrier()                                       # all ranks gather at once: symmetric NVLink load
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            dsm.gather(ids, out=out)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        assert dsm.device_error() == 0
        got = out[torch.from_numpy(check_idx).to(d.dev)].cpu().numpy()
        ok = d.all_true(np.array_equal(got, sfeat.feature_bytes(presets.FEAT_SEED, ids_np[check_idx], dim, dtype)))
        t = d.max(statistics.median(ts))
        algo = R * rb / t / 1e9
        t_roof = max(2 * R * rb / (peak * 1e9), (W - 1) / W * R * rb / (NVLINK_GBS * 1e9) if not d.shared_gpu else 0)
        cells.append({"dtype": dtype, "dim": dim, "row_bytes": rb, "ms": t * 1e3, "algo_gbs_per_gpu": algo,
                      "busbw_gbs_per_gpu": (W - 1) / W * algo, "hbm_gbs_read_plus_write": 2 * algo,
                      "frac_of_roofline": t_roof / t, "bound": "nvlink" if t_roof > 2 * R * rb / (peak * 1e9) else "hbm",
                      "rows_checked": len(check_idx), "bytes_ok": ok})
        del out
        d.barrier()
        dsm.destroy()
        torch.cuda.empty_cache()
        if not ok:
            raise SystemExit(f"sweep cell {dtype}:{dim}: gathered bytes differ from the generator")
    measured = [c for c in cells if "ms" in c]
    best = max(measured, key=lambda c: c["frac_of_roofline"]) if measured else {"algo_gbs_per_gpu": None,
                                                                                 "frac_of_roofline": None}
    if d.rank == 0:
        line = {"metric": f"feature gather AlgoBW per GPU vs HBM/NVLink roofline (config 4 sweep, W={W})",
                "value": best["algo_gbs_per_gpu"], "unit": "GB/s", "n_gpus": W, "steps": args.steps, "warmup": 3,
                "higher_is_better": True,
                "config": {"workload": "gather-sweep", "rows": n, "ids_per_rank": R, "ids": "uniform with replacement",
                           "sharding": f"row-sharded over {W} GPU(s), o(v) = v mod W", "l2": "flushed between gathers",
                           "gpus_visible": d.ndev, "exchange": "P2P loads (one kernel per GPU)"},
                "roofline": {"peak_hbm": peak, "peak_nvlink": NVLINK_GBS, "unit": "GB/s", "peak_source": peak_src,
                             "frac": best["frac_of_roofline"]},
                "cells": cells}
        emit(line, args)
    d.close()


def bench_latency(args):
    """NEXT #3 / PAPER.md Table I (L66-80): dependent 8 B load latency vs span (1..128 GB) through a DSM
    shard, one thread, `accesses` chained loads.  Rank 0 chases its own shard (local HBM) and, under
    torchrun with one GPU per rank, rank 1's shard (P2P over NVLink) -- the paper's P2P column.  With a
    single GPU the peer column is reported as not measurable."""
    import torch

    import paper_conf_sc_yanglql22_b200 as pkg
    from synth import gpu as sgpu
    from synth import presets
    d = Dist()
    free, _ = torch.cuda.mem_get_info()
    gib = 1 << 30
    spans = [int(float(s) * gib) // 512 * 512 for s in args.latency_spans.split(",")]
    spans = [sp for sp in spans if d.all_true(sp < 0.85 * free / max(1, d.world if d.shared_gpu else 1))]
    rows_per_rank = max(spans) // 512
    dsm = pkg.DSM(rows_per_rank * d.world, 0, 128, "fp32", 1, rank=d.rank, world_size=d.world, device=d.local,
                  allgather=d.ag)   # 512 B rows, filled with generator bits
    sgpu.fill_dsm_features_gpu(dsm, presets.FEAT_SEED, d.rank, d.world, 128, 0)
    torch.cuda.synchronize()
    d.barrier()
    res = []
    peer_ok = d.world > 1 and not d.shared_gpu
    if d.rank == 0:
        for sp in spans:
            row = {"span_gb": round(sp / gib, 4)}
            for name, r in (("local_ns", 0), ("peer_ns", 1)):
                if r >= d.world:
                    row[name] = None
                    continue
                dsm.chase(r, sp, 2000)                            # warm-up (TLB, clocks)
                row[name] = statistics.median(dsm.chase(r, sp, args.chase_accesses) for _ in range(3))
            if d.shared_gpu:
                row["peer_note"] = "ranks share one GPU: the 'peer' shard is local HBM"
            res.append(row)
    torch.cuda.synchronize()
    d.barrier()
    dsm.destroy()
    if d.rank == 0:
        line = {"metric": "dependent-load latency through a DSM shard (Table I analogue)",
                "value": res[-1]["peer_ns"] if peer_ok else res[-1]["local_ns"], "unit": "ns",
                "higher_is_better": False,
                "config": {"accesses": args.chase_accesses, "threads": 1, "n_gpus": d.world, "gpus_visible": d.ndev,
                           "value_is": "peer (NVLink P2P) latency at the largest span" if peer_ok else
                           "local HBM latency at the largest span (peer column not measurable: one GPU)",
                           "address_arithmetic": "2 dependent IMADs (~4 ns) per access",
                           "paper_A100_p2p_us": [1.35, 1.37, 1.43, 1.51, 1.56],
                           "paper_A100_um_us": [20.8, 29.6, 32.5, 35.3, 35.8]},
                "spans": res}
        emit(line, args)
    d.close()


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
    reorder, L178-180) on the same ids (config-4-style: uniform random ids per rank over the table of
    --config).  Under torchrun with one GPU per rank the all-to-alls run on NCCL over NVLink -- the
    paper's experiment.  At W=1 the all-to-alls are local copies: the ratio then only counts the extra
    memory passes and is labelled as NOT the paper's experiment.  Both outputs are byte-checked."""
    import torch

    from paper_conf_sc_yanglql22_b200 import loader
    from paper_conf_sc_yanglql22_b200.nccl_gather import DistributedGather
    from synth import features as sfeat
    from synth import presets, seeds
    d = Dist()
    p = presets.get(args.config)
    dsm, _ = loader.build_dsm(p, rank=d.rank, world=d.world, device=d.local, allgather=d.ag)
    dg = DistributedGather(dsm)  # (the CSR is not read here)
    ids_np = seeds.gather_ids(p.n, args.sweep_ids, presets.SEED_BASE, d.rank)
    ids = torch.from_numpy(ids_np).to(d.dev)
    out = torch.empty((ids.numel(), dsm.row_bytes), dtype=torch.uint8, device=d.dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=d.dev)
    check_idx = np.random.default_rng(d.rank).choice(len(ids_np), min(len(ids_np), 4096), replace=False)
    exp = sfeat.feature_bytes(presets.FEAT_SEED, ids_np[check_idx], p.feat_dim, p.feat_dtype)
    res = {}
    W = d.world
    for name, fn in (("p2p_one_kernel", lambda: dsm.gather(ids, out=out)),
                     ("distributed_five_step", lambda: dg.gather(ids, out=out))):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        ok = d.all_true(np.array_equal(out[torch.from_numpy(check_idx).to(d.dev)].cpu().numpy(), exp))
        ts = []
        for i in range(args.steps):
            flush.fill_(i & 0xFF)
            torch.cuda.synchronize()
            d.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        t = d.max(statistics.median(ts))
        algo = ids.numel() * dsm.row_bytes / t / 1e9
        res[name] = {"ms": t * 1e3, "algo_gbs_per_gpu": algo, "busbw_gbs_per_gpu": (W - 1) / W * algo,
                     "bytes_ok": ok, "rows_checked": len(check_idx)}
        if not ok:
            raise SystemExit(f"compare-gather: {name} bytes differ from the generator")
    assert dsm.device_error() == 0
    paper_exp = W > 1 and not d.shared_gpu
    if d.rank == 0:
        exch = "NCCL all-to-all over NVLink" if paper_exp else ("gloo via host (ranks share one GPU)" if W > 1 else
                                                               "local copy (W=1)")
        line = {"metric": "global gather: P2P (DSM, one kernel) vs distributed-memory five-step (Fig. 10 analogue)",
                "value": res["distributed_five_step"]["ms"] / res["p2p_one_kernel"]["ms"], "unit": "x (time ratio)",
                "higher_is_better": True, "n_gpus": W, "steps": args.steps,
                "is_paper_experiment": paper_exp,
                "note": None if paper_exp else "NOT the paper's experiment (needs one GPU per rank, W >= 2): the "
                        "all-to-alls are local, so the ratio only counts the five-step path's extra memory passes",
                "config": {"workload": p.name, "ids_per_rank": int(ids.numel()), "row_bytes": dsm.row_bytes,
                           "exchange": exch, "gpus_visible": d.ndev},
                "paper": "P2P gather >= 2x faster than the NCCL gather on 8x A100 (PAPER.md L297-305, Fig. 10)",
                "results": res}
        emit(line, args)
    torch.cuda.synchronize()
    d.barrier()
    dsm.destroy()
    d.close()


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
