#!/usr/bin/env python3
"""BASELINE configs[3]: n = 1..64, batch 1M -- interleaved vs canonical,
including the layout-conversion cost.

Per n (GPU, CUDA events, L2 flushed before every timed launch):
  * factor      -- batch_spotrf_interleaved (tuning table) on chunk-32 storage
  * to_inter    -- batch_canonical_to_interleaved (canonical [B][n*n] -> chunk 32)
  * to_canon    -- batch_interleaved_to_canonical
  * canonical path = to_inter + factor + to_canon
  * cusolver    -- context only: torch.linalg.cholesky_ex on a canonical [B, n, n]
                   batch (cuSOLVER batched potrf, the stand-in for the paper's
                   MAGMA comparison), upper triangle mirrored
Reports Gflop/s (n^3/3) and algorithmic GB/s (factor: 4n(n+1)+4 B/matrix;
conversion: 8n^2 B/matrix).  Writes JSON lines and a markdown table.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402


def timed(fn, prep, reps, flush):
    ts = []
    for _ in range(reps):
        prep()
        flush.fill_(1.0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", default="1-64")
    ap.add_argument("--batch", type=int, default=1 << 20)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/c4.jsonl")
    ap.add_argument("--md", default="gpurun_out/c4.md")
    ap.add_argument("--no-cusolver", action="store_true")
    a = ap.parse_args()
    lo, hi = (int(x) for x in a.n.split("-"))
    dev = torch.device("cuda", 0)
    B, chunk = a.batch, 32
    flush = torch.empty(512 << 18, dtype=torch.float32, device=dev)
    info = torch.empty(B, dtype=torch.int32, device=dev)
    rows = []
    f = open(a.out, "w")
    for n in range(lo, hi + 1):
        el = bsp.batch_interleaved_elems(n, B, chunk)
        inter = torch.empty(el, dtype=torch.float32, device=dev)
        pristine = torch.empty_like(inter)
        bsp.bspotrf_synth_generate(n, B, chunk, pristine, kind="dd", seed=2017)
        canon = torch.empty(B * n * n, dtype=torch.float32, device=dev)
        bsp.batch_interleaved_to_canonical(n, B, chunk, pristine, canon)
        t_fac = timed(lambda: bsp.batch_spotrf_interleaved(n, B, chunk, inter, info),
                      lambda: inter.copy_(pristine), a.reps, flush)
        t_in = timed(lambda: bsp.batch_canonical_to_interleaved(n, B, chunk, canon, inter),
                     lambda: None, a.reps, flush)
        t_out = timed(lambda: bsp.batch_interleaved_to_canonical(n, B, chunk, pristine, canon),
                      lambda: None, a.reps, flush)
        t_cus = None
        if not a.no_cusolver:
            try:
                M = canon.view(B, n, n)            # column-major matrices = row-major transposes; SPD symmetric
                work = torch.empty_like(M)
                t_cus = timed(lambda: torch.linalg.cholesky_ex(work), lambda: work.copy_(M), a.reps, flush)
            except Exception as ex:  # pragma: no cover
                t_cus = None
                print("cusolver failed", n, ex, flush=True)
        flops = B * n ** 3 / 3
        fb = B * (4 * n * (n + 1) + 4)
        cb = B * 8 * n * n
        t_canon = t_in + t_fac + t_out
        r = dict(n=n, batch=B, chunk=chunk, factor_ms=t_fac, to_inter_ms=t_in, to_canon_ms=t_out,
                 canonical_path_ms=t_canon, cusolver_ms=t_cus,
                 factor_gflops=flops / t_fac / 1e6, factor_gbs=fb / t_fac / 1e6,
                 convert_gbs=cb / ((t_in + t_out) / 2) / 1e6,
                 canonical_path_gflops=flops / t_canon / 1e6,
                 cusolver_gflops=(flops / t_cus / 1e6) if t_cus else None,
                 tuning=bsp.bspotrf_get_tuning(n, chunk).as_dict())
        rows.append(r)
        f.write(json.dumps(r) + "\n")
        f.flush()
        print(f"n={n} factor {t_fac:.4f} ms ({r['factor_gbs']:.0f} GB/s) canon-path {t_canon:.4f} ms "
              f"cusolver {t_cus}", flush=True)
        del inter, pristine, canon
        torch.cuda.empty_cache()
    with open(a.md, "w") as m:
        m.write("| n | factor ms | factor GB/s | factor Gflop/s | convert GB/s | canonical path ms "
                "(in+factor+out) | canonical Gflop/s | cuSOLVER ms | cuSOLVER Gflop/s |\n"
                "|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            cu = f"{r['cusolver_ms']:.4f} | {r['cusolver_gflops']:.0f}" if r["cusolver_ms"] else "- | -"
            m.write(f"| {r['n']} | {r['factor_ms']:.4f} | {r['factor_gbs']:.0f} | {r['factor_gflops']:.0f} | "
                    f"{r['convert_gbs']:.0f} | {r['canonical_path_ms']:.4f} | {r['canonical_path_gflops']:.0f} | "
                    f"{cu} |\n")


if __name__ == "__main__":
    main()
