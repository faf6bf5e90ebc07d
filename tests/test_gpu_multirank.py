"""W > 1 on one GPU: in-process virtual ranks (threads, same pid -> direct pointers)
and two processes sharing the GPU through real CUDA IPC handles.  Outputs must be
byte-identical to the oracle (and hence W-invariant, SURVEY.md 8(c) "W-invariance")."""

import os
import subprocess
import sys
import threading

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_yanglql22_b200 as pkg
from paper_conf_sc_yanglql22_b200 import loader
from synth import providers
from synth import graph, presets, seeds

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _create_all(p, W, flags=0, col32=None):
    ag = pkg.ThreadAllgather(W)
    out = [None] * W
    errs = []

    def run(r):
        try:
            out[r] = loader.build_dsm(p, rank=r, world=W, allgather=ag.for_rank(r), on_device=False, flags=flags,
                                      col32=col32)[0]
        except Exception as e:  # pragma: no cover
            errs.append(e)
    ths = [threading.Thread(target=run, args=(r,)) for r in range(W)]
    [t.start() for t in ths]
    [t.join() for t in ths]
    assert not errs, errs
    return out


def _destroy_all(dsms):
    ths = [threading.Thread(target=d.destroy) for d in dsms]
    [t.start() for t in ths]
    [t.join() for t in ths]


@pytest.mark.parametrize("W,placement", [(2, "dsm"), (3, "dsm"), (4, "dsm"), (8, "dsm"), (2, "csr-replicated"),
                                         (4, "csr-replicated"), (8, "csr-replicated"), (4, "dsm-col64"),
                                         (4, "csr-replicated-col64")])
def test_virtual_ranks_w_invariance(W, placement):
    """Every rank's batches are byte-identical to the oracle for the paper's placement (CSR and features
    row-sharded) and for the hybrid one (whole CSR on every rank, features sharded)."""
    p = presets.get("tiny")
    rp, col = graph.csr(p.graph())
    flags = pkg.WG_DSM_CSR_REPLICATED if placement.startswith("csr-replicated") else 0
    dsms = _create_all(p, W, flags, col32=not placement.endswith("col64"))
    rows = providers.host_row_provider(p.graph(), rp, col)
    feats = providers.host_feat_provider(p)
    for r, dsm in enumerate(dsms):
        assert dsm.shard_info(r)[0] == len(graph.shard_rows(p.n, r, W))
        if flags & pkg.WG_DSM_CSR_REPLICATED:
            lrp, lcol, _ = dsm.local_view()
            assert lrp.numel() == p.n + 1 and lcol.numel() == len(col)   # the whole CSR on every rank
        pipe = pkg.MiniBatchPipeline(dsm, p.fanouts, p.seeds_per_batch, with_pos=True, with_dup=True)
        for b in seeds.rank_batches(2 * W, r, W):
            S = seeds.seed_nodes(p.n, p.seeds_per_batch, presets.SEED_BASE, b)
            rs = seeds.rng_seed(presets.RNG_BASE, b)
            pipe.run(torch.from_numpy(S).cuda(), rs)
            torch.cuda.synchronize()
            ref = oracle.minibatch(rows, feats, S, p.fanouts, rs)
            for h in range(len(p.fanouts)):
                got, exp = pipe.result(h), ref["hops"][h]
                for k in ("row_ptr", "nbrs", "pos", "unique", "sub_col", "dup"):
                    assert np.array_equal(got[k], exp[k]), (W, r, b, h, k)
            assert np.array_equal(pipe.features(), ref["X"])
        assert dsm.device_error() == 0
    _destroy_all(dsms)


@pytest.mark.parametrize("mode", ["ipc", "ncclgather"])
def test_two_processes_cuda_ipc(mode):
    """torchrun-style 2 ranks (gloo for the handle allgather) on the SAME GPU: rank 1
    reads rank 0's shard through cudaIpcOpenMemHandle and vice versa."""
    port = 29500 + os.getpid() % 1000 + (7 if mode != "ipc" else 0)
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), WORLD_SIZE="2")
    procs = []
    for r in range(2):
        e = dict(env, RANK=str(r), LOCAL_RANK=str(r))
        procs.append(subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "mp_worker.py"), mode],
                                      env=e, stdout=subprocess.PIPE, stderr=subprocess.STDOUT))
    outs = [p.communicate(timeout=600)[0].decode() for p in procs]
    for p, o in zip(procs, outs):
        assert p.returncode == 0, o
        assert "PARITY OK" in o, o


def test_real_multi_gpu_processes():
    """W = min(device_count, 8) processes, rank r on its own GPU cuda:r: cross-device cudaIpcOpenMemHandle
    and NVLink P2P loads from the sampler and the gather, every array bit-exact against the oracle.
    Skips (visibly) on a one-GPU box, where the same-GPU IPC test below covers the host logic."""
    ndev = torch.cuda.device_count()
    if ndev < 2:
        pytest.skip(f"needs >= 2 GPUs for one process per GPU (this box has {ndev})")
    W = min(ndev, 8)
    port = 29400 + os.getpid() % 1000
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), WORLD_SIZE=str(W),
               LOCAL_WORLD_SIZE=str(W))
    procs = []
    for r in range(W):
        e = dict(env, RANK=str(r), LOCAL_RANK=str(r))
        procs.append(subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "mp_worker.py"), "ipc"],
                                      env=e, stdout=subprocess.PIPE, stderr=subprocess.STDOUT))
    outs = [p.communicate(timeout=900)[0].decode() for p in procs]
    for r, (p, o) in enumerate(zip(procs, outs)):
        assert p.returncode == 0, o
        assert "PARITY OK" in o and f"device cuda:{r}" in o, o


@pytest.mark.parametrize("placement", ["dsm", "csr-replicated", "replicas"])
def test_bench_torchrun_two_ranks(placement):
    """The driver's N>1 launch of bench.py (torchrun, one process per rank) on the one test GPU:
    every rank must reach the same collectives (max over ranks, barriers, collective destroy) and
    rank 0 prints one JSON line with the whole-job value."""
    import json
    port = 29600 + os.getpid() % 500 + {"dsm": 3, "csr-replicated": 5, "replicas": 0}[placement]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "3", "--warmup", "3", "--cpu-sample-s", "0", "--e2e-steps", "1",
           "--concurrency", "2", "--config", "tiny", "--placement", placement, "--north-star", ""]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["e2e"]["value"] > 0 and d["single_batch"]["value"] > 0
    assert d["config"]["parallelism"].startswith({"dsm": "dsm-w2", "csr-replicated": "csr-replicated-w2",
                                                  "replicas": "replicas-x2"}[placement])
    assert d["parity"]["ok"] is True and d["parity"]["ranks"] == 2 and d["parity"]["batches"] == 2


def _torchrun_line(args, port):
    import json
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "bench.py")] + args
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_sweep_two_ranks_byte_checked():
    """config-4 sweep under torchrun: the table row-sharded over 2 ranks, each gathering its own ids at once,
    every cell byte-checked against the generator on both ranks."""
    d = _torchrun_line(["--sweep", "--sweep-rows", "200000", "--sweep-ids", "20000", "--sweep-cells", "fp32:100,fp16:64",
                        "--steps", "2"], 29700 + os.getpid() % 300)
    assert d["n_gpus"] == 2 and len(d["cells"]) == 2
    for c in d["cells"]:
        assert c["bytes_ok"] is True and c["ms"] > 0 and c["busbw_gbs_per_gpu"] == c["algo_gbs_per_gpu"] / 2


def test_compare_gather_two_ranks():
    """NEXT #1 under torchrun (2 ranks sharing the GPU: gloo all-to-alls through the host): both gathers
    byte-checked, and the line says it is not the paper's experiment."""
    d = _torchrun_line(["--compare-gather", "--config", "tiny", "--sweep-ids", "20000", "--steps", "2"],
                       29720 + os.getpid() % 300)
    assert d["n_gpus"] == 2 and d["is_paper_experiment"] is False and d["note"]
    for r in d["results"].values():
        assert r["bytes_ok"] is True


def test_latency_two_ranks_peer_column():
    """Table I analogue under torchrun: rank 0 chases its own shard and rank 1's (labelled as local HBM when
    the ranks share a GPU)."""
    d = _torchrun_line(["--latency", "--latency-spans", "0.0625", "--chase-accesses", "2000"], 29740 + os.getpid() % 300)
    row = d["spans"][0]
    assert row["local_ns"] > 0 and row["peer_ns"] > 0 and "peer_note" in row
