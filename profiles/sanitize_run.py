"""Workload for the compute-sanitizer pass (SURVEY.md section 4 tier 4 / section 5): the tiny config
(configs[0]) through every path of libwg.so that the product uses, small enough to run under
memcheck / racecheck / synccheck / initcheck in minutes.

  1. the fused pipeline (wg_sample_hop + incremental wg_gather_rows), eager and as a CUDA graph replay;
  2. two workspace forks on two concurrent streams (the relabel side streams, the scan ring);
  3. the separate ops (wg_sample_neighbors, wg_append_unique, wg_gather) and a fanout > 32 hop;
  4. W = 2 in-process virtual ranks (peer pointers in the shard view);
  5. g-SpMM forward / backward on the last hop.
Every result is compared with the oracle, so a sanitizer-clean run is also a parity-green run.
"""

import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sc_yanglql22_b200 as pkg  # noqa: E402
from paper_conf_sc_yanglql22_b200 import loader  # noqa: E402
from synth import graph, presets, providers, seeds  # noqa: E402


def check_pipe(pipe, ref, fanouts):
    for h in range(len(fanouts)):
        got, exp = pipe.result(h), ref["hops"][h]
        for k in ("row_ptr", "nbrs", "unique", "sub_col"):
            assert np.array_equal(got[k], exp[k]), (h, k)
    assert np.array_equal(pipe.features(), ref["X"])


def main():
    torch.cuda.set_device(0)
    p = presets.get("tiny")
    rp, col = graph.csr(p.graph())
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    batches = [0, 1, 2]
    refs = {}
    for b in batches:
        S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
        refs[b] = (S, seeds.rng_seed(presets.RNG_BASE, b))
        refs[b] = refs[b] + (oracle.minibatch(rows, feats, S, p.fanouts, refs[b][1]),)

    dsm, _ = loader.build_dsm(p, on_device=False)
    # 1. fused pipeline, eager then graph replay
    pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_dup=True)
    for b in batches:
        S, rs, ref = refs[b]
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        check_pipe(pipe, ref, p.fanouts)
    pipe.capture()
    for b in batches:
        S, rs, ref = refs[b]
        pipe.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        check_pipe(pipe, ref, p.fanouts)
    print("fused pipeline + graph replay OK", flush=True)

    # 2. two forks on two streams, concurrently
    forks = [dsm.fork(), dsm.fork()]
    pipes = [pkg.MiniBatchPipeline(f, p.fanouts, p.seeds_per_batch) for f in forks]
    sts = [torch.cuda.Stream(), torch.cuda.Stream()]
    for b in batches:
        for j in range(2):
            S, rs, _ = refs[(b + j) % len(batches)]
            with torch.cuda.stream(sts[j]):
                pipes[j].run(torch.from_numpy(S).pin_memory(), rs, stream=sts[j])
        torch.cuda.synchronize()
        for j in range(2):
            check_pipe(pipes[j], refs[(b + j) % len(batches)][2], p.fanouts)
    print("two forks on two streams OK", flush=True)

    # 3. separate ops + fanout > 32
    S, rs, ref = refs[0]
    t = torch.from_numpy(S).cuda()
    rpo, nb, pos, ne = dsm.sample_neighbors(t, p.fanouts[0], rs, 0, with_pos=True)
    e = int(ne.item())
    assert np.array_equal(nb[:e].cpu().numpy(), ref["hops"][0]["nbrs"])
    U, nU, sc, dup = dsm.append_unique(t, nb[:e], with_dup=True)
    u = int(nU.item())
    assert np.array_equal(U[:u].cpu().numpy(), ref["hops"][0]["unique"])
    X = dsm.gather(U[:u])
    torch.cuda.synchronize()
    assert np.array_equal(X[:u].cpu().numpy(), feats(U[:u].cpu().numpy())[1][
        np.searchsorted(feats(U[:u].cpu().numpy())[0], U[:u].cpu().numpy())])
    big = dsm.sample_neighbors(t[:64], 40, rs, 0)
    torch.cuda.synchronize()
    ad_ptr, ad = rows(S[:64])
    _, exp_nbrs, _ = oracle.sample_hop(ad_ptr, ad, S[:64], 40, rs, 0)
    assert np.array_equal(big[1][: int(big[3].item())].cpu().numpy(), exp_nbrs)
    print("separate ops + fanout 40 OK", flush=True)

    # 5. g-SpMM on the last hop of batch 0 (pipeline with dup counts)
    from paper_conf_sc_yanglql22_b200 import layers
    S, rs, ref = refs[0]
    pipe.run(torch.from_numpy(S).cuda(), rs)
    torch.cuda.synchronize()
    last, prev = pipe.hops[-1], pipe.hops[-2]
    T = int(prev["num_unique"].item())
    E = int(last["num_edges"].item())
    U_ = int(last["num_unique"].item())
    Xf = pipe.X_rows[:U_].contiguous().view(torch.float32).reshape(U_, p.feat_dim)
    y = layers.spmm_mean_forward(last["row_ptr"][:T + 1], last["sub_col"][:E], Xf)
    dx = layers.spmm_mean_backward(last["row_ptr"][:T + 1], last["sub_col"][:E], last["dup"][:U_],
                                   torch.ones_like(y), U_)
    torch.cuda.synchronize()
    assert torch.isfinite(y).all() and torch.isfinite(dx).all()
    print("g-SpMM OK", flush=True)
    for f in forks:
        f.destroy()
    assert dsm.device_error() == 0
    dsm.destroy()

    # 4. W = 2 virtual ranks
    W = 2
    ag = pkg.ThreadAllgather(W)
    out = [None] * W

    def mk(r):
        out[r] = loader.build_dsm(p, rank=r, world=W, allgather=ag.for_rank(r), on_device=False)[0]
    ths = [threading.Thread(target=mk, args=(r,)) for r in range(W)]
    [x.start() for x in ths]
    [x.join() for x in ths]
    for r in range(W):
        pv = pkg.MiniBatchPipeline(out[r], p.fanouts, p.seeds_per_batch)
        S, rs, ref = refs[r]
        pv.run(torch.from_numpy(S).cuda(), rs)
        torch.cuda.synchronize()
        check_pipe(pv, ref, p.fanouts)
        assert out[r].device_error() == 0
    ths = [threading.Thread(target=d.destroy) for d in out]
    [x.start() for x in ths]
    [x.join() for x in ths]
    print("W=2 virtual ranks OK", flush=True)
    print("SANITIZE WORKLOAD OK", flush=True)


if __name__ == "__main__":
    main()
