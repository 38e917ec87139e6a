#!/usr/bin/env python3
"""A/B of the fused canonical factorization (batch_spotrf_canonical): one
group per warp (BSPOTRF_CANON_PF=0) vs persistent warps with the next group's
copies in flight (=1), per n at 1M matrices; median of 5 launches, input
regenerated and L2 flushed before each.  One JSON line per (n, pf)."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

B = 1 << 20
flush = torch.empty(128 << 20, dtype=torch.float32, device="cuda")
inter = torch.empty(bsp.batch_interleaved_elems(20, B, 32), device="cuda")
canon = torch.empty(B * 400, device="cuda")
info = torch.empty(B, dtype=torch.int32, device="cuda")
cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
for n in range(1, bsp.CANON_MAX_N + 1):
    iv, cv = inter[:bsp.batch_interleaved_elems(n, B, 32)], canon[:B * n * n]
    for pf in ("0", "1"):
        os.environ["BSPOTRF_CANON_PF"] = pf
        ts = []
        cnt.zero_()
        for rep in range(6):
            bsp.bspotrf_synth_generate(n, B, 32, iv, kind="dd", seed=2017)
            bsp.batch_interleaved_to_canonical(n, B, 32, iv, cv)
            flush.fill_(rep)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            bsp.batch_spotrf_canonical(n, B, cv, info, nfailed=cnt)
            b.record()
            torch.cuda.synchronize()
            if rep:
                ts.append(a.elapsed_time(b))
        ms = statistics.median(ts)
        byt = B * (4 * n * (n + 1) + 4)
        print(json.dumps({"n": n, "pf": int(pf), "ms": round(ms, 4), "gbs": round(byt / ms / 1e6, 1),
                          "gflops": round(B * n ** 3 / 3 / ms / 1e6, 1), "fails": int(cnt.item())}), flush=True)
