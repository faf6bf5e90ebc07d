#!/usr/bin/env python
"""DRAM traffic of the throughput pass (bench pass B) as ONE workload: P products-shaped batch
pipelines (workspace forks) captured on P forked streams into one CUDA graph, so

    ncu --graph-profiling graph --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
        python profiles/ncu_passb.py [both|prep|gather] [P]

reports the bytes the concurrent batches really move (ncu's per-kernel numbers are cold-cache and
serialised).  Without ncu it prints the graph's event-timed duration (median of 20 replays)."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yanglql22_b200 as pkg  # noqa: E402
from paper_conf_sc_yanglql22_b200 import loader  # noqa: E402
from synth import presets, seeds  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "both"
P = int(sys.argv[2]) if len(sys.argv) > 2 else 8
p = presets.get(os.environ.get("CONFIG", "products"))
dsm, _ = loader.build_dsm(p)
handles = [dsm] + [dsm.fork() for _ in range(P - 1)]
GP, SP, MP = (int(os.environ.get(k, 0)) for k in ("PRIO_GATHER", "PRIO_SIDE", "PRIO_MAIN"))
# gathers at the throughput occupancy bench pass B / MiniBatchLoader use (GATHER_OCC, 0 = occupancy max)
OCC = int(os.environ.get("GATHER_OCC", pkg.pipeline.THROUGHPUT_GATHER_OCCUPANCY))
for h in handles:
    h.set_gather_occupancy(OCC)
pipes = [pkg.MiniBatchPipeline(h, p.fanouts, p.seeds_per_batch, gather_priority=GP, side_priority=SP)
         for h in handles]
S = p.seeds_per_batch
for j, pl in enumerate(pipes):   # eager warm-up; fills X / hop buffers for the gather-only mode
    pl.run(torch.from_numpy(seeds.seed_nodes(p.n, S, presets.SEED_BASE, j)).cuda(), seeds.rng_seed(presets.RNG_BASE, j))
torch.cuda.synchronize()

g = torch.cuda.CUDAGraph()
cap = torch.cuda.Stream()
streams = [torch.cuda.Stream(priority=MP) for _ in range(P)]
cap.wait_stream(torch.cuda.current_stream())
with torch.cuda.graph(g, stream=cap):
    for j, pl in enumerate(pipes):   # fork all P batches first, then join (they run concurrently)
        streams[j].wait_stream(cap)
        if mode == "gather":
            pl.enqueue_gather(streams[j])
        else:
            pl.enqueue(streams[j], gather=(mode == "both"))
    for j in range(P):
        cap.wait_stream(streams[j])
torch.cuda.current_stream().wait_stream(cap)
torch.cuda.synchronize()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
ts = []
for i in range(int(os.environ.get("REPS", 20))):
    for j, pl in enumerate(pipes):   # new seeds every replay (inputs resident in HBM)
        pl.set_inputs(torch.from_numpy(seeds.seed_nodes(p.n, S, presets.SEED_BASE, 100 + i * P + j)).cuda(),
                      seeds.rng_seed(presets.RNG_BASE, 100 + i * P + j))
    flush.fill_(i & 0xFF)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
assert all(h.device_error() == 0 for h in handles)
rows = sum(int(pl.hops[-1]["num_unique"].item()) for pl in pipes)
t = statistics.median(ts)
print(f"mode={mode} P={P} prio(g,s,m)={GP},{SP},{MP} graph_ms_median={t:.4f} per_batch_us={1e3 * t / P:.1f} "
      f"seeds_per_s={P * S / (t / 1e3):.0f} rows_gathered_last={rows}", flush=True)
