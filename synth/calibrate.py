"""Fit d_min so that the generated CSR lands near a target size (SURVEY.md 8(d)
"Fitting d_min").  Run once; the results are frozen into ``presets.py``.

    python -m synth.calibrate
"""

import numpy as np

from .graph import GraphSpec, rows

TARGETS = {
    # name: (n, target CSR entries)
    "tiny": (10_000, 200_000),
    "products": (2_450_000, 124_000_000),
    "papers100m": (111_000_000, 3_200_000_000),
    "mag240m": (244_000_000, 3_400_000_000),
}


def mean_degree(n, d_min, gs, sample):
    spec = GraphSpec(n=n, d_min=d_min, graph_seed=gs)
    ptr, _ = rows(spec, sample)
    return ptr[-1] / len(sample)


def fit(n, target_e, gs, sample_size=200_000, iters=30):
    if n <= sample_size:
        sample = np.arange(n, dtype=np.int64)
    else:
        sample = np.linspace(0, n - 1, sample_size).astype(np.int64)
    want = target_e / n
    lo, hi = 0.1, want
    for _ in range(iters):
        mid = 0.5 * (lo + hi)
        if mean_degree(n, mid, gs, sample) < want:
            lo = mid
        else:
            hi = mid
    return 0.5 * (lo + hi)


if __name__ == "__main__":
    from .presets import GRAPH_SEED
    for name, (n, e) in TARGETS.items():
        dm = fit(n, e, GRAPH_SEED)
        print(f"{name}: d_min={dm:.6f} (mean target {e / n:.3f})", flush=True)
