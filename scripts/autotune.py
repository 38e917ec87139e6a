#!/usr/bin/env python3
"""Autotuning sweep on the B200 (§II.D).

Exhaustive over the B200 axes (north star (4)):
  * chunk size C            -- 32, 64, 128, 256, 512 and 0 (simple interleaved)
  * variant = unroll depth / staging:
      REG   full unroll, registers only             (paper: fully unrolled, n_b = n)
      SMEM  full unroll, left panel of S columns in shared memory, staged by
            TMA bulk copy (staging 1) or per-thread cp.async (staging 2)
      TILE  tile ops unrolled, outer loops rolled, NB x NB tiles
            (paper: partially unrolled top-looking, n_b = NB)
      PANEL/PTMEM/RTMA/RTMAP  see include/bspotrf.h
      QTM   P threads per matrix (4, 8), TMEM columns per CTA (256, 512), n > 32
      RCW   8 warps per 32 matrices, CTAs per SM (1, 2), n > 32
      REGV  4 adjacent matrices per thread, 128-bit accesses, n <= 8
  * threads per block       -- 32..256
  * L1 / shared carveout     -- --carveouts (percent of max shared memory; 0 =
                               driver default): Table I's sixth parameter,
                               PAPER.md:216,407
Each point: regenerate the batch in place (device generator), flush L2, time
ONE launch with CUDA events; median of --reps.  Every point is also checked
(failure count 0 on SPD input).  Appends JSON lines (resumable).

    python scripts/autotune.py --n 1-32 --chunks 32,64,128,256,512,0 --out gpurun_out/sweep.jsonl

The full candidate space needs the sweep build (BSPOTRF_SWEEP=1 python -m
paper_conf_ipps_gatesklpd17_b200.build); the default build records the points
it lacks as error -7.
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_gatesklpd17_b200 as bsp  # noqa: E402

REG, SMEM, TILE = bsp.VARIANT_REG, bsp.VARIANT_SMEM, bsp.VARIANT_TILE


def parse_range(s):
    out = []
    for part in s.split(","):
        if "-" in part:
            a, b = part.split("-")
            out += list(range(int(a), int(b) + 1))
        else:
            out.append(int(part))
    return out


PANEL = bsp.VARIANT_PANEL
PTMEM = bsp.VARIANT_PTMEM
RTMA = bsp.VARIANT_RTMA


def candidates(n, chunk):
    c = []
    if n <= 24:
        for tpb in (32, 64, 128, 256):
            c.append(dict(variant=REG, threads_per_block=tpb, param=0, staging=0))
    if 11 <= n <= 17:
        c.append(dict(variant=REG, threads_per_block=128, param=12, staging=0))
    if 11 <= n <= 14:
        c.append(dict(variant=REG, threads_per_block=128, param=16, staging=0))
    if 20 <= n <= 32:
        for s in range(4, n - 7, 4):
            if n - s > 16:
                continue
            if chunk in (32, 64, 128):
                c.append(dict(variant=PANEL, threads_per_block=0, param=s, staging=1))
            for tpb in (32, 64):
                c.append(dict(variant=PANEL, threads_per_block=tpb, param=s, staging=2))
    if 4 <= n <= 20 and chunk == 32:
        for w in (2, 4):
            c.append(dict(variant=RTMA, threads_per_block=0, param=w, staging=1))
            c.append(dict(variant=bsp.VARIANT_RTMAP, threads_per_block=0, param=w, staging=1))
    if 24 <= n <= 44:
        sys.path.insert(0, os.path.join(ROOT, "scripts"))
        import gen_instances
        for s in gen_instances.ptmem_s_values(n):
            if chunk == 32:
                c.append(dict(variant=PTMEM, threads_per_block=128, param=s, staging=1))
                if n <= 32:
                    c.append(dict(variant=PTMEM, threads_per_block=128, param=s, staging=3))
            c.append(dict(variant=PTMEM, threads_per_block=128, param=s, staging=2))
    if 17 <= n <= 32:
        for s in (n - 16, n - 14, n - 12):
            if not (2 <= s <= n - 2):
                continue
            if chunk in (32, 64, 128):
                c.append(dict(variant=SMEM, threads_per_block=0, param=s, staging=1))
            for tpb in (32, 64, 128):
                c.append(dict(variant=SMEM, threads_per_block=tpb, param=s, staging=2))
    if n <= 16:
        sys.path.insert(0, os.path.join(ROOT, "scripts"))
        import gen_instances
        for m, fast in gen_instances.regx_combos(n):
            for tpb in (64, 128):
                c.append(dict(variant=bsp.VARIANT_REGX, threads_per_block=tpb, param=m, staging=int(fast)))
    if n <= 8:
        for tpb in (64, 128):
            c.append(dict(variant=bsp.VARIANT_REGV, threads_per_block=tpb, param=0, staging=0))
    if 33 <= n <= 64:
        sys.path.insert(0, os.path.join(ROOT, "scripts"))
        import gen_instances
        for p_, cols, pre in gen_instances.QTM_COMBOS:
            if gen_instances.qtm_fits(n, p_, cols, pre):
                c.append(dict(variant=bsp.VARIANT_QTM, threads_per_block=128, param=p_,
                              staging=gen_instances.qtm_staging(cols, pre)))
    sys.path.insert(0, os.path.join(ROOT, "scripts"))
    import gen_instances
    if n in gen_instances.RCW_N:
        for k in gen_instances.rcw_ncta(n):
            c.append(dict(variant=bsp.VARIANT_RCW, threads_per_block=256, param=k, staging=0))
    if n in gen_instances.RCW16_N:
        c.append(dict(variant=bsp.VARIANT_RCW16, threads_per_block=512, param=0, staging=0))
    if n in gen_instances.RCWD_N:
        c.append(dict(variant=bsp.VARIANT_RCWD, threads_per_block=288, param=0, staging=0))
    if n in gen_instances.RCWP_N:
        for prm in gen_instances.rcwp_params(n):
            c.append(dict(variant=bsp.VARIANT_RCWP, threads_per_block=256, param=prm, staging=0))
    for nb in (2, 4, 8):
        if nb <= n or nb == 2:
            for tpb in (64, 128, 256):
                c.append(dict(variant=TILE, threads_per_block=tpb, param=nb, staging=0))
    return c


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", default="1-32")
    ap.add_argument("--chunks", default="32,64,128,256,512,0")
    ap.add_argument("--batch", type=int, default=1 << 20)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/sweep.jsonl")
    ap.add_argument("--kind", default="dd")
    ap.add_argument("--skip-from", action="append", default=[],
                    help="JSONL files whose points are already measured")
    ap.add_argument("--variants", default="1,2,3,4,5,6,7,8,10,11,12,13,14")   # 9 (REGX) on request
    ap.add_argument("--carveouts", default="0", help="e.g. 0,1,25,50,100")
    ap.add_argument("--only", default=None,
                    help="JSON list of tunings to measure instead of candidates() (e.g. table rows)")
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    done = set()
    for path in [a.out] + a.skip_from:
        if os.path.exists(path):
            for line in open(path):
                r = json.loads(line)
                done.add((r["n"], r["chunk"], r["variant"], r["threads_per_block"], r["param"], r["staging"],
                          r.get("carveout", 0)))
    variants = {int(v) for v in a.variants.split(",")}
    carveouts = [int(v) for v in a.carveouts.split(",")]
    dev = torch.device("cuda", 0)
    B = a.batch
    flush = torch.empty(512 << 18, dtype=torch.float32, device=dev)   # 512 MB > L2
    info = torch.empty(B, dtype=torch.int32, device=dev)
    cnt = torch.zeros(1, dtype=torch.int32, device=dev)
    f = open(a.out, "a")
    t_start = time.time()
    for n in parse_range(a.n):
        for chunk in [int(x) for x in a.chunks.split(",")]:
            elems = bsp.batch_interleaved_elems(n, B, chunk)
            A = torch.empty(elems, dtype=torch.float32, device=dev)
            pristine = torch.empty_like(A)
            bsp.bspotrf_synth_generate(n, B, chunk, pristine, kind=a.kind, seed=2017)
            cands = candidates(n, chunk)
            if a.only:
                cands = [dict(variant=t["variant"], threads_per_block=t["threads_per_block"],
                              param=t["param"], staging=t["staging"])
                         for t in json.loads(a.only) if t.get("n", n) == n and t.get("chunk", chunk) == chunk]
            cands = [dict(t, carveout=cv) for t in cands for cv in carveouts]
            for t in cands:
                if t["variant"] not in variants:
                    continue
                key = (n, chunk, t["variant"], t["threads_per_block"], t["param"], t["staging"], t["carveout"])
                if key in done:
                    continue
                times = []
                err = None
                for _ in range(a.reps):
                    A.copy_(pristine)
                    flush.fill_(1.0)
                    cnt.zero_()
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record()
                    try:
                        bsp.batch_spotrf_interleaved_ex(n, B, chunk, A, info, nfailed=cnt, tune=t)
                    except bsp.BspotrfError as ex:
                        err = ex.code
                        break
                    e1.record()
                    torch.cuda.synchronize()
                    times.append(e0.elapsed_time(e1))
                    if int(cnt.item()) != 0:
                        err = "nonzero failure count on SPD input"
                        break
                rec = dict(n=n, chunk=chunk, batch=B, **t)
                if err is not None:
                    rec["error"] = err
                else:
                    ms = statistics.median(times)
                    rec.update(ms=round(ms, 5), gbs=round(B * (4 * n * (n + 1) + 4) / ms / 1e6, 1),
                               gflops=round(B * n ** 3 / 3 / ms / 1e6, 1), reps=times)
                f.write(json.dumps(rec) + "\n")
                f.flush()
            del A, pristine
            torch.cuda.empty_cache()
        print(f"n={n} done at {time.time() - t_start:.0f}s", flush=True)


if __name__ == "__main__":
    main()
