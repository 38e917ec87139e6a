#!/usr/bin/env python3
"""Launch the tuning-table winner once per n (batch 1M, chunk 32) so that one
`ncu --metrics ...` pass can attribute DRAM throughput and FP32-pipe use to the
sweep's choices (north star (4): choices justified by ncu counters).

    ncu --metrics <list> --csv --log-file gpurun_out/ncu_winners.csv \\
        python scripts/ncu_winners.py --n 1-32
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", default="1-32")
ap.add_argument("--batch", type=int, default=1 << 20)
ap.add_argument("--chunk", type=int, default=32)
a = ap.parse_args()
lo, hi = (int(x) for x in a.n.split("-"))
info = torch.empty(a.batch, dtype=torch.int32, device="cuda")
for n in range(lo, hi + 1):
    A = torch.empty(bsp.batch_interleaved_elems(n, a.batch, a.chunk), device="cuda")
    bsp.bspotrf_synth_generate(n, a.batch, a.chunk, A, kind="dd", seed=2017)
    bsp.batch_spotrf_interleaved(n, a.batch, a.chunk, A, info)
    torch.cuda.synchronize()
    print(n, bsp.bspotrf_get_tuning(n, a.chunk).as_dict(), flush=True)
    del A
