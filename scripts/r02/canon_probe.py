#!/usr/bin/env python3
"""One fused canonical factorization per n (1M matrices) -- an ncu target."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

B = 1 << 20
for n in [int(x) for x in (sys.argv[1:] or ["16"])]:
    inter = torch.empty(bsp.batch_interleaved_elems(n, B, 32), device="cuda")
    bsp.bspotrf_synth_generate(n, B, 32, inter, kind="dd", seed=2017)
    canon = torch.empty(B * n * n, device="cuda")
    bsp.batch_interleaved_to_canonical(n, B, 32, inter, canon)
    info = torch.empty(B, dtype=torch.int32, device="cuda")
    bsp.batch_spotrf_canonical(n, B, canon, info)
    torch.cuda.synchronize()
    del inter, canon
    torch.cuda.empty_cache()
print("ok")
