"""The five BASELINE.json configurations as named presets.

d_min values were produced by ``python -m synth.calibrate`` (host bisection on a
200k-node sample) and refined with the exact CSR size by ``python -m
synth.calibrate_gpu`` (log: profiles/r01/calibrate_gpu.log); they are frozen here so
that every run generates the same graphs (E = 200,000 / ~124.0M / ~3.20B / ~3.40B).
"""

from dataclasses import dataclass, field
from typing import List

from .graph import GraphSpec

GRAPH_SEED = 0x5EED_600D
FEAT_SEED = 0xFEA7_5EED
SEED_BASE = 1_000_003          # PCG64(base + b) for the seed nodes of batch b
RNG_BASE = 0x0123_4567_89AB_CDEF


@dataclass(frozen=True)
class Preset:
    name: str
    n: int
    target_e: int
    d_min: float
    feat_dim: int
    feat_dtype: str
    fanouts: List[int] = field(default_factory=list)
    seeds_per_batch: int = 1024
    note: str = ""

    def graph(self) -> GraphSpec:
        return GraphSpec(n=self.n, d_min=self.d_min, graph_seed=GRAPH_SEED)


PRESETS = {
    "tiny": Preset("tiny", 10_000, 200_000, 5.529218, 32, "fp32", [10, 5], 512,
                   "configs[0]: synthetic power-law graph 10k nodes / 200k edges, 32-dim fp32, [10,5], 512 seeds"),
    "products": Preset("products", 2_450_000, 124_000_000, 13.252141, 100, "fp32", [15, 10, 5], 1024,
                       "configs[1]: ogbn-products-shaped, 100-dim fp32, [15,10,5], 1024 seeds/GPU"),
    "papers100m": Preset("papers100m", 111_000_000, 3_200_000_000, 7.54903, 128, "fp32", [15, 10, 5], 1024,
                         "configs[2]: ogbn-papers100M-shaped, 128-dim fp32, [15,10,5], 1024 seeds/GPU"),
    "mag240m": Preset("mag240m", 244_000_000, 3_400_000_000, 3.694334, 768, "fp16", [25, 15], 1024,
                      "configs[4]: MAG240M-shaped, 768-dim fp16, [25,15], 1024 seeds/GPU"),
}


def get(name: str) -> Preset:
    return PRESETS[name]
