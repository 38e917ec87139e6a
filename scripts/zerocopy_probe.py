#!/usr/bin/env python3
"""e2e design probe: factor PINNED HOST interleaved storage in place with each
kernel variant (zero-copy: the kernel's loads/stores cross PCIe), vs the copy
pipeline.  Prints ms and PCIe GB/s each way."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp

out = []
for n, B in ((16, 1 << 20), (32, 1 << 20)):
    chunk = 32
    el = bsp.batch_interleaved_elems(n, B, chunk)
    d = torch.empty(el, device="cuda")
    bsp.bspotrf_synth_generate(n, B, chunk, d, kind="dd", seed=2017)
    pristine = d.cpu()
    del d
    hA = torch.empty(el).pin_memory()
    hinfo = torch.empty(B, dtype=torch.int32).pin_memory()
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    hb = bsp.batch_spotrf_host_bytes(n, B, chunk)
    cands = [dict(variant=1, threads_per_block=tpb, param=mw, staging=0) for tpb, mw in ((128, 0), (256, 0), (128, 12))] + \
            [dict(variant=6, threads_per_block=0, param=w, staging=1) for w in (2, 4)] + \
            [dict(variant=5, threads_per_block=128, param=16, staging=st) for st in (1, 2)] + \
            [dict(variant=4, threads_per_block=0, param=16, staging=1), dict(variant=3, threads_per_block=64, param=4, staging=0)]
    for t in cands:
        ts = []
        ok = True
        for rep in range(3):
            hA.copy_(pristine)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            try:
                bsp.batch_spotrf_interleaved_ex(n, B, chunk, hA.data_ptr(), hinfo.data_ptr(), nfailed=cnt, tune=t)
                torch.cuda.synchronize()
            except Exception as ex:
                ok = False
                out.append(dict(n=n, tune=t, error=str(ex)))
                break
            ts.append(time.perf_counter() - t0)
        if ok:
            ms = min(ts) * 1e3
            bad = int((hinfo != 0).sum())
            out.append(dict(n=n, tune=t, ms=round(ms, 3), pcie_gbs=round(hb / ms / 1e6, 2), bad_info=bad))
        print(out[-1], flush=True)
    for slab in (0, 4096 * 16, 4096 * 64):
        ts = []
        for rep in range(3):
            hA.copy_(pristine)
            t0 = time.perf_counter()
            bsp.batch_spotrf_interleaved_host(n, B, chunk, hA, hinfo, slab=slab)
            ts.append(time.perf_counter() - t0)
        ms = min(ts) * 1e3
        out.append(dict(n=n, host_call_slab=slab, ms=round(ms, 3), pcie_gbs=round(hb / ms / 1e6, 2)))
        print(out[-1], flush=True)
json.dump(out, open("gpurun_out/zerocopy_probe.json", "w"), indent=1)
