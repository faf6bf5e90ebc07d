"""Single-batch critical path inside one CUDA graph (diagnostics, not a bench line): cumulative graphs of
hops [0], [0,1], [0,1,2] without gather, the shipped graph (incremental gather), and a chain of trivial
kernels for the per-launch floor.  L2 flushed before each replay (outside the events); medians of 30."""
import os
import statistics
import sys

sys.path.insert(0, os.getcwd())
import torch

import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import presets, seeds

wl = sys.argv[1] if len(sys.argv) > 1 else "products"
p = presets.get(wl)
dsm, _ = loader.build_dsm(p, flags=int(os.environ.get("WG_FLAGS", "0"), 0))
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream()


NOFLUSH = os.environ.get("NOFLUSH") == "1"


def timed(run, n=30, warm=3):
    ts = []
    for i in range(n + warm):
        if not NOFLUSH:
            flush.fill_(i & 0xFF)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        run(i)
        b.record(st)
        torch.cuda.synchronize()
        if i >= warm:
            ts.append(a.elapsed_time(b) * 1e3)
    return statistics.median(ts)


res = {}
for H in range(1, len(p.fanouts) + 1):
    for gather in (False, True):
        if gather and H < len(p.fanouts):
            continue
        pipe = pkg.MiniBatchPipeline(dsm, p.fanouts[:H], p.seeds_per_batch)

        def setin(i, pipe=pipe):
            pipe.set_inputs(torch.from_numpy(seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, i)).cuda(),
                            seeds.rng_seed(presets.RNG_BASE, i))
        setin(0)
        pipe.enqueue(gather=gather)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        s = torch.cuda.Stream()
        s.wait_stream(st)
        with torch.cuda.graph(g, stream=s):
            pipe.enqueue(gather=gather)
        st.wait_stream(s)
        ins = [torch.from_numpy(seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, i)).cuda() for i in range(40)]

        def run(i, pipe=pipe, g=g, ins=ins):
            pipe.set_inputs(ins[i % 40], seeds.rng_seed(presets.RNG_BASE, i))
            g.replay()
        res[f"hops{H}{'+gather' if gather else ''}"] = timed(run)
        res[f"hops{H}{'+gather' if gather else ''}_replay_only"] = timed(lambda i, g=g: g.replay())
        if H == 1:
            res["set_inputs_only"] = timed(lambda i, pipe=pipe, ins=ins: pipe.set_inputs(
                ins[i % 40], seeds.rng_seed(presets.RNG_BASE, i)))
        del g, pipe

# per-launch floor: 12 trivial kernels in a graph
x = torch.zeros(16, device="cuda")
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
s.wait_stream(st)
with torch.cuda.graph(g, stream=s):
    for _ in range(12):
        x.add_(1)
st.wait_stream(s)
res["12_trivial_kernels"] = timed(lambda i: g.replay())
res["empty"] = timed(lambda i: None)
print(wl, "noflush" if NOFLUSH else "flush", "flags", os.environ.get("WG_FLAGS", "0"), " ".join(f"{k}={v:.1f}us" for k, v in res.items()), flush=True)
