#!/usr/bin/env python3
"""PCIe ceiling for the e2e path: pinned host <-> device cudaMemcpy bandwidth,
each direction alone and both at once (two streams)."""
import json
import time

import torch

N = 1 << 30
h = torch.empty(N // 4, dtype=torch.float32).pin_memory()
h2 = torch.empty(N // 4, dtype=torch.float32).pin_memory()
d = torch.empty(N // 4, dtype=torch.float32, device="cuda")
d2 = torch.empty(N // 4, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def t(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


h2d = N / t(lambda: d.copy_(h, non_blocking=True)) / 1e9
d2h = N / t(lambda: h.copy_(d, non_blocking=True)) / 1e9


def both():
    with torch.cuda.stream(s1):
        d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2):
        h2.copy_(d2, non_blocking=True)


bi = t(both)
print(json.dumps({"h2d_gbs": round(h2d, 2), "d2h_gbs": round(d2h, 2),
                  "bidirectional_each_way_gbs": round(N / bi / 1e9, 2)}))
