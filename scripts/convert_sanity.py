#!/usr/bin/env python3
"""Minimal layout-conversion run for compute-sanitizer (memcheck) triage."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402
from oracle import layout  # noqa: E402

for n in (1, 2, 3, 16):
    for chunk in (32, 0):
        batch = 517
        canon = np.random.default_rng(n).standard_normal((batch, n * n)).astype(np.float32)
        src = torch.from_numpy(canon).cuda()
        dst = torch.zeros(bsp.batch_interleaved_elems(n, batch, chunk), device="cuda")
        print("n", n, "chunk", chunk, "src", hex(src.data_ptr()), src.numel() * 4, "dst", hex(dst.data_ptr()),
              dst.numel() * 4, flush=True)
        bsp.batch_canonical_to_interleaved(n, batch, chunk, src, dst)
        torch.cuda.synchronize()
        ok = np.array_equal(dst.cpu().numpy(), layout.to_interleaved(n, chunk, canon))
        back = torch.zeros_like(src)
        bsp.batch_interleaved_to_canonical(n, batch, chunk, dst, back)
        torch.cuda.synchronize()
        print("  ok", ok, np.array_equal(back.cpu().numpy(), canon), flush=True)
