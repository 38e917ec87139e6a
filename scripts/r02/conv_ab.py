#!/usr/bin/env python3
"""A/B timing of the layout-conversion paths (v2 vs v3, forced through
BSPOTRF_CONVERT_PATH) per n at batch 1M, chunk 32: median of 5 single launches
per direction, L2 flushed (512 MB write) before each, CUDA events on the
current stream.  Prints one JSON line per (n, path)."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

B = int(os.environ.get("CONV_AB_BATCH", 1 << 20))
chunk = 32
def parse(spec):
    out = []
    for part in spec.split(","):
        a, _, b = part.partition("-")
        out += list(range(int(a), int(b or a) + 1))
    return out


ns = parse(sys.argv[1] if len(sys.argv) > 1 else "6-64")
paths = (sys.argv[2] if len(sys.argv) > 2 else "v2,v3").split(",")
flush = torch.empty(128 << 20, dtype=torch.float32, device="cuda")
peak = 6545.9
for n in ns:
    el = bsp.batch_interleaved_elems(n, B, chunk)
    inter = torch.empty(el, device="cuda")
    bsp.bspotrf_synth_generate(n, B, chunk, inter, kind="dd", seed=2017)
    canon = torch.empty(B * n * n, device="cuda")
    nbytes = 2 * 4 * B * n * n
    for p in paths:
        os.environ["BSPOTRF_CONVERT_PATH"] = p
        t = {0: [], 1: []}
        for rep in range(6):
            for d in (1, 0):
                flush.fill_(rep)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                if d == 1:
                    bsp.batch_interleaved_to_canonical(n, B, chunk, inter, canon)
                else:
                    bsp.batch_canonical_to_interleaved(n, B, chunk, canon, inter)
                b.record()
                torch.cuda.synchronize()
                if rep:
                    t[d].append(a.elapsed_time(b))
        r = {"n": n, "path": p}
        for d, name in ((1, "to_canon"), (0, "to_inter")):
            ms = statistics.median(t[d])
            r[name + "_gbs"] = round(nbytes / ms / 1e6, 1)
            r[name + "_frac"] = round(nbytes / ms / 1e6 / peak, 3)
        print(json.dumps(r), flush=True)
    del inter, canon
    torch.cuda.empty_cache()
