#!/usr/bin/env python
"""Per-kernel device times of one mini-batch, measured with CUDA events between the
kernels of a captured graph replay is not possible, so this replays the batch eagerly
with an event after every op (launch gaps included) -- warm caches, no profiler.

    python profiles/stage_times.py [--config products] [--batches 20]
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yanglql22_b200 as pkg  # noqa: E402
from paper_conf_sc_yanglql22_b200 import loader  # noqa: E402
from synth import presets, seeds  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="products")
    ap.add_argument("--batches", type=int, default=20)
    ap.add_argument("--flush", action="store_true")
    ap.add_argument("--graph", action="store_true", help="capture the ops + events as one CUDA graph")
    args = ap.parse_args()
    p = presets.get(args.config)
    dsm, _ = loader.build_dsm(p)
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, fused=False)
    st = torch.cuda.current_stream()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda") if args.flush else None
    names = []
    for h in range(len(p.fanouts)):
        names += [f"hop{h}.sample+compact", f"hop{h}.unique(insert+flag+relabel)"]
    names.append("gather")
    acc = {n: [] for n in names}
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(len(names) + 1)]

    def enqueue():
        evs[0].record(torch.cuda.current_stream())
        tgt, tcap, tn = pipe.seeds, pipe.max_seeds, pipe.n_seeds
        e = 1
        cur = torch.cuda.current_stream()
        for h, m in enumerate(p.fanouts):
            bb = pipe.hops[h]
            dsm.sample_neighbors(tgt, m, 0, h, n_targets_dev=tn, seed_dev=pipe.rng_seed, out_row_ptr=bb["row_ptr"],
                                 out_nbrs=bb["nbrs"], out_num_edges=bb["num_edges"], cap=tcap)
            evs[e].record(cur)
            e += 1
            dsm.append_unique(tgt, bb["nbrs"], n_targets=tcap, n_nbrs=pipe.E_cap[h], n_targets_dev=tn,
                              n_nbrs_dev=bb["num_edges"], out_unique=bb["unique"], out_num_unique=bb["num_unique"],
                              out_sub_col=bb["sub_col"])
            evs[e].record(cur)
            e += 1
            tgt, tcap, tn = bb["unique"], pipe.U_cap[h], bb["num_unique"]
        pipe.enqueue_gather()
        evs[e].record(cur)

    g = None
    for b in range(args.batches + 3):
        S = torch.from_numpy(seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)).cuda()
        pipe.set_inputs(S, seeds.rng_seed(presets.RNG_BASE, b))
        if flush is not None:
            flush.fill_(b & 0xFF)
        if args.graph and b == 1:
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                enqueue()
        if g is not None:
            g.replay()
        else:
            enqueue()
        torch.cuda.synchronize()
        if b >= 3:
            for i, n in enumerate(names):
                acc[n].append(evs[i].elapsed_time(evs[i + 1]) * 1e3)
    tot = 0
    for n in names:
        m = statistics.median(acc[n])
        tot += m
        print(f"{m:8.1f} us  {n}")
    print(f"{tot:8.1f} us  total (eager, separate ops, launch gaps included)")
    dsm.destroy()


if __name__ == "__main__":
    main()
