"""Worker for the multi-process tests (one process per rank; env RANK/WORLD_SIZE/
MASTER_ADDR/MASTER_PORT).  Mode "ipc": rank r drives cuda:(r % device_count) -- its own GPU on a
multi-GPU box, all ranks on cuda:0 on a one-GPU box -- the DSM handles are exchanged over gloo and
opened with cudaIpcOpenMemHandle (a peer on another GPU is read over NVLink); mode "gloo-host":
CPU-only check of the host-side collective plumbing."""

import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402


def main():
    mode = sys.argv[1]
    dist.init_process_group("gloo", init_method="env://")
    rank, world = dist.get_rank(), dist.get_world_size()
    if mode == "gloo-host":
        from paper_conf_sc_yanglql22_b200.dsm import TorchDistAllgather
        ag = TorchDistAllgather()
        import ctypes
        send = (ctypes.c_uint8 * 16)(*([rank + 1] * 16))
        recv = (ctypes.c_uint8 * (16 * world))()
        assert ag(ctypes.addressof(send), ctypes.addressof(recv), 16, None) == 0
        got = bytes(recv)
        assert got == b"".join(bytes([r + 1] * 16) for r in range(world)), got
        assert ag(None, None, 0, None) == 0     # barrier
        print("GLOO OK", flush=True)
    elif mode == "ipc":
        import oracle
        import paper_conf_sc_yanglql22_b200 as pkg
        from paper_conf_sc_yanglql22_b200 import loader
        from synth import providers
        from synth import graph, presets, seeds
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        print(f"rank {rank} on device cuda:{dev}", flush=True)
        p = presets.get("tiny")
        ag = pkg.TorchDistAllgather()
        dsm, _ = loader.build_dsm(p, rank=rank, world=world, device=dev, allgather=ag, on_device=False)
        rp, col = graph.csr(p.graph())
        rows = providers.host_row_provider(p.graph(), rp, col)
        feats = providers.host_feat_provider(p)
        pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
        for b in seeds.rank_batches(4, rank, world):
            S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
            rs = seeds.rng_seed(presets.RNG_BASE, b)
            pipe.run(torch.from_numpy(S).cuda(), rs)
            torch.cuda.synchronize()
            ref = oracle.minibatch(rows, feats, S, p.fanouts, rs)
            for h in range(len(p.fanouts)):
                got, exp = pipe.result(h), ref["hops"][h]
                for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                    assert np.array_equal(got[k], exp[k]), (rank, b, h, k)
            assert np.array_equal(pipe.features(), ref["X"])
        assert dsm.device_error() == 0
        dsm.destroy()
        print("PARITY OK", flush=True)
    elif mode == "ncclgather":
        import oracle
        import paper_conf_sc_yanglql22_b200 as pkg
        from paper_conf_sc_yanglql22_b200 import loader
        from synth import providers
        from paper_conf_sc_yanglql22_b200.nccl_gather import DistributedGather
        from synth import features, presets
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        p = presets.get("tiny")
        ag = pkg.TorchDistAllgather()
        dsm, _ = loader.build_dsm(p, rank=rank, world=world, device=dev, allgather=ag, on_device=False)
        ids = np.random.default_rng(rank).integers(0, p.n, 7000).astype(np.int64)
        out = DistributedGather(dsm).gather(torch.from_numpy(ids).cuda())
        direct = dsm.gather(torch.from_numpy(ids).cuda())
        torch.cuda.synchronize()
        exp = features.feature_bytes(presets.FEAT_SEED, ids, p.feat_dim, p.feat_dtype)
        assert np.array_equal(out[:len(ids)].cpu().numpy(), exp)
        assert np.array_equal(direct[:len(ids)].cpu().numpy(), exp)
        dsm.destroy()
        print("PARITY OK", flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
