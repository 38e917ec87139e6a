#!/usr/bin/env python3
"""Small-n ceiling (C4, n = 1..8 at batch 1M): what a plain device copy with the
SAME traffic achieves, timed like the factorization (CUDA events around one
launch, L2 flushed before each).  The factorization of n x n matrices reads and
writes 4n(n+1)/2 bytes per matrix plus a 4-byte info store; a copy of
bytes/2 (read) into another buffer (write) moves the same bytes.  The ratio
factorization / copy says how far the kernel is from the launch + DRAM-latency
floor that a 1M batch of tiny matrices sits on."""
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


def timed(fn, prep, reps=9):
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


rows = []
for n in range(1, 9):
    fb = B * (4 * n * (n + 1) + 4)                    # algorithmic bytes (read + write)
    A = torch.empty(bsp.batch_interleaved_elems(n, B, chunk), device="cuda")
    A0 = torch.empty_like(A)
    bsp.bspotrf_synth_generate(n, B, chunk, A0, kind="dd", seed=2017)
    tf = timed(lambda: bsp.batch_spotrf_interleaved(n, B, chunk, A, info), lambda: A.copy_(A0))
    src = torch.ones(fb // 8, device="cuda")          # fb/2 bytes read, fb/2 written
    dst = torch.empty_like(src)
    tc = timed(lambda: dst.copy_(src), lambda: None)
    te = timed(lambda: None, lambda: None)            # empty event pair
    rows.append(dict(n=n, bytes=fb, factor_ms=tf, copy_ms=tc, empty_events_ms=te,
                     factor_gbs=fb / tf / 1e6, copy_gbs=fb / tc / 1e6, factor_over_copy=tc / tf))
    print(json.dumps(rows[-1]), flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(rows, open("gpurun_out/small_n_ceiling.json", "w"), indent=1)
