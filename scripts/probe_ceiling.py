#!/usr/bin/env python3
"""Access-pattern ceiling: the null factorization (REG's exact loads/stores,
no arithmetic) vs the factorization, n in {4, 8, 16, 20}, batch 1M, chunk 32."""
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
out = []


def timed(fn, prep, reps=7):
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


for n in (4, 8, 16, 20):
    A = torch.empty(bsp.batch_interleaved_elems(n, B, chunk), device="cuda")
    A0 = torch.empty_like(A)
    bsp.bspotrf_synth_generate(n, B, chunk, A0, kind="dd", seed=2017)
    fb = B * (4 * n * (n + 1) + 4)
    for tpb in (64, 128, 256):
        t = timed(lambda: bsp.bspotrf_probe_copy_lower(n, B, A, info, tpb=tpb), lambda: A.copy_(A0))
        out.append(dict(n=n, kind="null-factorization", tpb=tpb, ms=t, gbs=fb / t / 1e6))
        print(json.dumps(out[-1]), flush=True)
    t = timed(lambda: bsp.batch_spotrf_interleaved(n, B, chunk, A, info), lambda: A.copy_(A0))
    out.append(dict(n=n, kind="factorization (table)", ms=t, gbs=fb / t / 1e6,
                    tuning=bsp.bspotrf_get_tuning(n, chunk).as_dict()))
    print(json.dumps(out[-1]), flush=True)
    del A, A0
json.dump(out, open("gpurun_out/probe_ceiling.json", "w"), indent=1)
