"""N > 1 with the real kernel on one GPU (north star (5)).

The build pod has one GPU, so two ranks share cuda:0 under the gloo backend
(NCCL refuses two ranks on one device); everything else is the multi-GPU path:
chunk-aligned slices of global indices (multi_gpu.RankBatch), the
factorization kernel's fused failure count on each rank, and the one
all-reduce of that count.  The global count must equal the enumerated
failure plan (pin P10), and sampled matrices of every slice must pass the
oracle.  A second test drives bench.py itself under torchrun with two ranks.
"""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch.multiprocessing as mp

import synth

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, Bg, chunk, P, q):
    try:
        import torch
        import torch.distributed as dist

        import oracle
        from oracle import checks, layout
        from paper_conf_ipps_gatesklpd17_b200 import multi_gpu
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                          WORLD_SIZE=str(world), LOCAL_RANK="0")
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        rb = multi_gpu.RankBatch(n, Bg, chunk, kind="dd", seed=2017, fail_seed=2018,
                                 fail_period=P, device=torch.device("cuda", 0))
        rb.regenerate()
        rb.factor()
        torch.cuda.synchronize()
        local = int(rb.nfailed.item())                 # the kernel's own fused count
        total = rb.global_failures()                   # the one collective
        # sampled oracle check of this rank's slice (global indices -> same matrices)
        idx = np.unique(np.concatenate([np.arange(0, rb.count, max(1, rb.count // 300)),
                                        np.arange(max(0, rb.count - 40), rb.count)]))
        A = synth.generate(n, "dd", 2017, (rb.b0 + idx).astype(np.uint64), upper="mirror",
                           fail_seed=2018, fail_period=P)
        L64, info64 = oracle.potrf(n, A)
        flat = rb.A.cpu().numpy()
        ii, jj = np.tril_indices(n)
        got = np.zeros((idx.size, n * n), np.float32)
        for t, b in enumerate(idx):
            offs = layout.offset(n, rb.count, chunk, b, ii, jj)
            got[t, ii + jj * n] = flat[offs]
            got[t, jj + ii * n] = np.where(ii != jj, A[t, jj + ii * n], got[t, ii + jj * n])
        ginfo = rb.info.cpu().numpy()[idx]
        r = checks.accept(n, A, got, ginfo, L64, info64)
        q.put((rank, rb.b0, rb.count, local, total, bool(r["ok"].all()), None))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, None, None, None, None, False, repr(e)))


@pytest.mark.parametrize("n,Bg,chunk", [(32, 200_000, 32), (16, 100_003, 0)])
def test_two_ranks_one_gpu_kernel_count_allreduce(n, Bg, chunk):
    world, P = 2, 1009
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, Bg, chunk, P, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert all(r[6] is None for r in res), res
    expected = synth.expected_fail_count(n, 2018, P, 0, Bg)
    assert expected > 0
    for rank, b0, cnt, local, total, ok, _ in res:
        assert local == synth.expected_fail_count(n, 2018, P, b0, b0 + cnt)
        assert total == expected
        assert ok
    assert sum(r[2] for r in res) == Bg


def test_bench_two_ranks_under_torchrun():
    """bench.py's N > 1 path (RankBatch slices, per-step all-reduce of the count,
    max-over-ranks timing, strong scaling on c5's global batch) end to end."""
    port = _free_port()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), "bench.py",
           "--gpus", "2", "--workload", "c5", "--batch", str(1 << 20), "--steps", "4",
           "--warmup", "3", "--dist-backend", "gloo", "--same-device", "--per-n", "none",
           "--no-cpu-baseline", "--e2e-steps", "1"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["value"] > 0
    assert d["config"]["batch_per_gpu"] == 1 << 19
    assert d["e2e"]["value"] > 0
