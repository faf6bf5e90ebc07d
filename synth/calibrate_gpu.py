"""Refine d_min on the device with the exact CSR size (full generation per trial).

    python -m synth.calibrate_gpu papers100m mag240m
"""
import sys
import time

import torch

from . import presets
from .graph import GraphSpec
from .gpu import shard_csr_gpu


def exact_e(n, d_min, gs):
    rp, col = shard_csr_gpu(GraphSpec(n=n, d_min=d_min, graph_seed=gs), 0, 1, torch.device("cuda", 0))
    e = int(rp[-1].item())
    del rp, col
    torch.cuda.empty_cache()
    return e


if __name__ == "__main__":
    for name in sys.argv[1:]:
        p = presets.get(name)
        lo, hi = p.d_min * 0.85, p.d_min * 1.05
        for it in range(14):
            mid = 0.5 * (lo + hi)
            t = time.time()
            e = exact_e(p.n, mid, presets.GRAPH_SEED)
            print(f"{name} it{it} d_min={mid:.6f} E={e} ({time.time() - t:.1f}s)", flush=True)
            if e < p.target_e:
                lo = mid
            else:
                hi = mid
        print(f"RESULT {name} d_min={0.5 * (lo + hi):.6f}", flush=True)
