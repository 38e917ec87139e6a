#!/usr/bin/env python3
"""Small launches of the round-2 kernels (fused canonical factorization,
conversion v3, RCWP at a runtime chunk) -- the target of compute-sanitizer
memcheck / racecheck / synccheck runs (scripts/r02/gpu_job18.sh)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

B = 4096 + 37
for n in (7, 16, 20):                                     # CANON
    inter = torch.empty(bsp.batch_interleaved_elems(n, B, 32), device="cuda")
    bsp.bspotrf_synth_generate(n, B, 32, inter, kind="dd", seed=1, fail_seed=2, fail_period=7)
    canon = torch.empty(B * n * n, device="cuda")
    bsp.batch_interleaved_to_canonical(n, B, 32, inter, canon)
    info = torch.empty(B, dtype=torch.int32, device="cuda")
    bsp.batch_spotrf_canonical(n, B, canon, info)
for n in (13, 14, 63):                                    # conversion v3 (interleaved -> canonical)
    inter = torch.empty(bsp.batch_interleaved_elems(n, B, 32), device="cuda")
    bsp.bspotrf_synth_generate(n, B, 32, inter, kind="dd", seed=1)
    canon = torch.empty(B * n * n, device="cuda")
    bsp.batch_interleaved_to_canonical(n, B, 32, inter, canon)
for n, chunk in ((57, 0), (64, 96)):                      # RCWP, runtime-chunk prefetch
    A = torch.empty(bsp.batch_interleaved_elems(n, B, chunk), device="cuda")
    bsp.bspotrf_synth_generate(n, B, chunk, A, kind="dd", seed=1)
    info = torch.empty(B, dtype=torch.int32, device="cuda")
    bsp.batch_spotrf_interleaved_ex(n, B, chunk, A, info,
                                    tune={"variant": bsp.VARIANT_RCWP, "threads_per_block": 256, "param": 0,
                                          "staging": 0})
torch.cuda.synchronize()
print("ok")
