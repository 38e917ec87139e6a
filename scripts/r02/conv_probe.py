#!/usr/bin/env python3
"""One launch of each layout conversion direction at given n (1M matrices,
chunk 32) -- the target of an ncu capture (scripts/r02/gpu_job3.sh)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

B = 1 << 20
for n in [int(x) for x in (sys.argv[1:] or ["63", "64"])]:
    inter = torch.empty(bsp.batch_interleaved_elems(n, B, 32), dtype=torch.float32, device="cuda")
    canon = torch.empty(B * n * n, dtype=torch.float32, device="cuda")
    bsp.bspotrf_synth_generate(n, B, 32, inter, kind="dd", seed=1)
    bsp.batch_interleaved_to_canonical(n, B, 32, inter, canon)
    bsp.batch_canonical_to_interleaved(n, B, 32, canon, inter)
    torch.cuda.synchronize()
    del inter, canon
    torch.cuda.empty_cache()
print("ok")
