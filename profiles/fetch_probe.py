"""DRAM fetch-granularity probe for the gather (run under ncu; see fetch_probe.sh).

For each row size, gathers R uniform-random rows of a table of n rows (pitch = row bytes
rounded up to 64 B, as the DSM lays them out) into a dense or 32 B-pitched output, once per
cell, with L2 flushed before.  ncu's dram__bytes_read.sum per launch / R is the DRAM bytes
fetched per gathered row; comparing it with the row's sectors / 64 B chunks / 128 B lines
tells which granule the L2 fetches at.  WG_L2_FETCH=<bytes> sets cudaLimitMaxL2FetchGranularity
first (cuda-python)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_sc_yanglql22_b200 as pkg  # noqa: E402
from synth import gpu as sgpu  # noqa: E402
from synth import presets, seeds  # noqa: E402


def main():
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    g = os.environ.get("WG_L2_FETCH")
    if g:
        from cuda.bindings import runtime as rt
        print("set L2 fetch granularity", g, rt.cudaDeviceSetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity, int(g)))
    n = int(os.environ.get("PROBE_ROWS", 8_000_000))
    R = int(os.environ.get("PROBE_IDS", 1_000_000))
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    ids = torch.from_numpy(seeds.gather_ids(n, R, presets.SEED_BASE, 0)).to(dev)
    begin = torch.zeros(1, dtype=torch.int64, device=dev)
    end = torch.full((1,), R, dtype=torch.int64, device=dev)
    cells = [(8, 0), (16, 0), (24, 0), (32, 0), (64, 0), (96, 0), (100, 0), (100, 1), (104, 0), (112, 0), (128, 0)]
    for dim, pitched in cells:   # fp32 dims: 32 B .. 512 B rows
        rb = dim * 4
        dsm = pkg.DSM(n, 0, dim, "fp32", 1, device=0)
        _, _, fv = dsm.local_view()
        sgpu.fill_dsm_features_gpu(dsm, presets.FEAT_SEED, 0, 1, dim, 0)
        pitch = dsm.out_pitch() if pitched else rb
        out = torch.empty((R, pitch), dtype=torch.uint8, device=dev)
        for _ in range(2):
            dsm.gather_rows(ids, R, begin, end, out)
        flush.fill_(1)
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_push(f"rb{rb}_p{pitch}")
        dsm.gather_rows(ids, R, begin, end, out)   # the measured launch (3rd of the cell)
        torch.cuda.nvtx.range_pop()
        torch.cuda.synchronize()
        print(f"cell rb={rb} feat_pitch={fv.stride(0)} out_pitch={pitch} R={R}", flush=True)
        del out, fv
        dsm.destroy()
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
