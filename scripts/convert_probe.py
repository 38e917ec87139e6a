#!/usr/bin/env python3
"""One launch per (n, direction) of the layout-conversion kernels at batch 1M,
chunk 32 -- a short command for an ncu capture (scripts/gpu_round25.sh)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

B, chunk = 1 << 20, 32
for n in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "31,32").split(",")]:
    el = bsp.batch_interleaved_elems(n, B, chunk)
    inter = torch.empty(el, device="cuda")
    bsp.bspotrf_synth_generate(n, B, chunk, inter, kind="dd", seed=2017)
    canon = torch.empty(B * n * n, device="cuda")
    for _ in range(2):
        bsp.batch_interleaved_to_canonical(n, B, chunk, inter, canon)
        bsp.batch_canonical_to_interleaved(n, B, chunk, canon, inter)
    torch.cuda.synchronize()
    del inter, canon
