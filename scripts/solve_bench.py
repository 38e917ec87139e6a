#!/usr/bin/env python3
"""SPOSV / SPOTRS throughput on B200: batch 1M, chunk 32.
Algorithmic bytes: fused SPOSV = factor bytes + 2*4*n*nrhs (B read + X written);
SPOTRS = 2 passes over L (2 * 2n(n+1)) + 2*4*n*nrhs."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

B, chunk = 1 << 20, 32
flush = torch.empty(512 << 18, device="cuda")
info = torch.empty(B, dtype=torch.int32, device="cuda")
rows = []


def timed(fn, prep, reps=5):
    ts = []
    for _ in range(reps):
        prep()
        flush.fill_(1.0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)


for n in (4, 8, 16, 20, 24, 28, 32, 36, 40, 44):
    for nrhs in (1, 4):
        A = torch.empty(bsp.batch_interleaved_elems(n, B, chunk), device="cuda")
        A0 = torch.empty_like(A)
        bsp.bspotrf_synth_generate(n, B, chunk, A0, kind="dd", seed=2017)
        Bm = torch.randn(bsp.batch_interleaved_rhs_elems(n, nrhs, B, chunk), device="cuda")
        B0 = Bm.clone()
        t_sposv = timed(lambda: bsp.batch_sposv_interleaved(n, nrhs, B, chunk, A, Bm, info),
                        lambda: (A.copy_(A0), Bm.copy_(B0)))
        bsp.batch_spotrf_interleaved(n, B, chunk, A, info)
        t_potrs = timed(lambda: bsp.batch_spotrs_interleaved(n, nrhs, B, chunk, A, Bm),
                        lambda: Bm.copy_(B0))
        fb = 4 * n * (n + 1) + 4
        rb = 8 * n * nrhs
        r = dict(n=n, nrhs=nrhs, sposv_ms=round(t_sposv, 4), potrs_ms=round(t_potrs, 4),
                 sposv_gbs=round(B * (fb + rb) / t_sposv / 1e6, 1),
                 potrs_gbs=round(B * (2 * 2 * n * (n + 1) + rb) / t_potrs / 1e6, 1),
                 fused=bool((n <= 20 and nrhs <= 4) or (24 <= n <= 44 and nrhs == 1)))
        rows.append(r)
        print(json.dumps(r), flush=True)
        del A, A0, Bm, B0
json.dump(rows, open("gpurun_out/solve_bench.json", "w"), indent=1)
