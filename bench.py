#!/usr/bin/env python3
"""Benchmark: batched FP32 SPOTRF (lower, in place) on interleaved storage.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload c2|c1|c3|c2i|c4n<N>] [--n --batch --chunk --kind]

A "step" is one pass of the hot path (addressing, load,
pivot/sqrt, column scale, rank-1 update, store + info + fused failure count,
tuning-table dispatch; plus the failure-count all-reduce when N > 1) over one
batch of synthetic SPD matrices already resident in HBM: exactly one launch of
our factorization kernel per step.  Every step factors a DIFFERENT
pre-generated buffer (the factorization is in place), each larger than L2,
so no step sees another's data in cache; when K exceeds the buffers that fit
in HBM the pool is regenerated between groups of steps, outside the timed
region.  Timing: CUDA events on the launching stream, barrier +
synchronize on both sides, max over ranks.  Default workload: BASELINE.json
configs[2] (n=32, batch=4M per GPU, chunk 32, ALS-shaped), the largest
single-GPU config -- weak scaling over GPUs.  The line also carries the "vs n"
half of the metric ("per_n": every n in 1..64 at 1M matrices, the table's
kernel, fraction of measured HBM bandwidth, the canonical path with layout
conversion; "per_n_large_batch": n <= 8 at 64M matrices), measured after the
timed region.

Prints ONE JSON line (rank 0).  Metric unit: Gflop/s with n^3/3 flops per
matrix; the HBM side of the metric is in "hbm_gbs" and
"roofline".
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "batched SPOTRF Gflop/s and HBM GB/s vs n (interleaved), 1/2/4/8 B200"

WORKLOADS = {
    "c2": dict(n=16, batch=1 << 20, chunk=32, kind="dd",
               desc="BASELINE configs[1]: n=16, batch=1M (1048576) per GPU, chunked interleaved "
                    "C=32, diagonally dominant SPD"),
    "c2i": dict(n=16, batch=1 << 20, chunk=0, kind="dd",
                desc="configs[1] variant: n=16, batch=1M per GPU, simple (fully) interleaved"),
    "c1": dict(n=8, batch=16384, chunk=32, kind="dd",
               desc="BASELINE configs[0]: n=8, batch=16384, chunk 32 (launch/latency-bound)"),
    "c3": dict(n=32, batch=1 << 22, chunk=32, kind="als",
               desc="BASELINE configs[2]: n=32, batch=4M, ALS-shaped regularised Gram, chunk 32"),
    "c5": dict(n=32, batch=1 << 25, chunk=32, kind="dd", global_batch=True, fail_period=1009,
               desc="BASELINE configs[4]: n=32, batch=32M (33554432) GLOBAL split over the GPUs "
                    "(strong scaling), DD SPD with injected failures (1 in 1009), failure-count "
                    "all-reduce"),
}

FLAG_NAMES = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
              0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
              0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
              0x100: "display_clock_setting"}


def flops_per_matrix(n):          # "the standard formula, N^3/3"
    return n ** 3 / 3.0


def bytes_per_matrix(n):          # lower triangle read + written, FP32, + int32 info
    return 4 * n * (n + 1) + 4


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c3")
    ap.add_argument("--n", type=int)
    ap.add_argument("--batch", type=int)
    ap.add_argument("--chunk", type=int)
    ap.add_argument("--kind")
    ap.add_argument("--tune", help='JSON tuning override, e.g. {"variant":2,"param":18,...}')
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--cpu-seconds", type=float, default=8.0,
                    help="target CPU time of the cpu_baseline sample")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--max-pool-gb", type=float, default=120.0)
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for N > 1 (gloo: test mode, see --same-device)")
    ap.add_argument("--same-device", action="store_true",
                    help="test mode: every rank uses cuda:0 (needs --dist-backend gloo)")
    ap.add_argument("--per-n", default="1-64",
                    help="n values of the per-n block (1M matrices, chunk 32; n <= 8 also at 64M), "
                         "e.g. 1-32,48,64, or none")
    return ap.parse_args()


def workload(a):
    if a.workload.startswith("c4n"):
        w = dict(n=int(a.workload[3:]), batch=1 << 20, chunk=32, kind="dd",
                 desc=f"BASELINE configs[3] point: n={a.workload[3:]}, batch=1M, chunk 32")
    else:
        w = dict(WORKLOADS[a.workload])
    for k in ("n", "batch", "chunk", "kind"):
        v = getattr(a, k)
        if v is not None:
            w[k] = v
            w["desc"] = w["desc"] + f" [override {k}={v}]"
    w["name"] = a.workload
    return w


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def traffic_from_profiles(w):
    """dram read+write bytes per launch of the factor kernel from a committed
    ncu --set full capture summary (profiles/ncu_traffic.json), if any."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(p))
        key = f"n{w['n']}_b{w['batch']}_c{w['chunk']}"
        return d[key]["dram_bytes_per_launch"]
    except Exception:
        return None


# --------------------------------------------------------------------- CPU side
def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_oracle_rate(n, kind, target_s, max_batch, seed=2017, cores=None):
    """Time the oracle (as it stands) on a bounded sample of the workload:
    matrices 0..S-1 (S <= batch), repeated in passes until ~target_s seconds
    of wall time have been spent factoring (input generation excluded)."""
    import numpy as np

    import oracle
    import synth
    cores = cores or oracle.default_threads()
    probe = min(max_batch, max(256, int(2e6 / max(1.0, flops_per_matrix(n)))))
    A = synth.generate(n, kind, seed, np.arange(probe, dtype=np.uint64))
    t0 = time.perf_counter()
    oracle.potrf(n, A, nthreads=cores)
    dt = max(time.perf_counter() - t0, 1e-6)
    S = int(min(max_batch, 1 << 20, max(probe, probe * target_s / dt)))
    A = synth.generate(n, kind, seed, np.arange(S, dtype=np.uint64))
    total_t, passes = 0.0, 0
    while total_t < target_s or passes == 0:
        t0 = time.perf_counter()
        oracle.potrf(n, A, nthreads=cores)
        total_t += time.perf_counter() - t0
        passes += 1
    gflops = S * passes * flops_per_matrix(n) / total_t / 1e9
    return dict(value=round(gflops, 4), unit="Gflop/s", cores=cores, kind="oracle",
                sample=f"matrices 0..{S - 1} of the workload ({S} of {max_batch}) x {passes} "
                       f"pass(es), canonical FP32 in, FP64 Algorithm 1 (oracle/cholesky.c), "
                       f"{cores} threads, {total_t:.2f} s factoring; generation excluded")


def run_reference(a, w):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import numpy as np

    import oracle
    import synth
    n, kind = w["n"], w["kind"]
    cores = oracle.default_threads()
    probe = min(w["batch"], 4096)
    model = cpu_model()
    A = synth.generate(n, kind, 2017, np.arange(probe, dtype=np.uint64))
    t0 = time.perf_counter()
    oracle.potrf(n, A, nthreads=cores)
    dt = max(time.perf_counter() - t0, 1e-6)
    budget = 90.0 / max(1, a.steps + a.warmup)           # whole run within ~1.5 min
    S = int(min(w["batch"], max(probe, probe * budget / dt)))
    A = synth.generate(n, kind, 2017, np.arange(S, dtype=np.uint64))
    for _ in range(a.warmup):
        oracle.potrf(n, A, nthreads=cores)
    times = []
    for _ in range(a.steps):
        t0 = time.perf_counter()
        oracle.potrf(n, A, nthreads=cores)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    value = S * a.steps * flops_per_matrix(n) / tot / 1e9
    sample = (f"each step: matrices 0..{S - 1} of the workload ({S} of {w['batch']}), canonical "
              f"FP32 in, FP64 Algorithm 1 (oracle/cholesky.c), {cores} host threads")
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "Gflop/s",
        "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": round(1e3 * tot / a.steps, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": config_of(w, a),
        "cpu_baseline": {"value": round(value, 4), "unit": "Gflop/s", "cores": cores,
                         "kind": "oracle", "sample": sample, "cpu_model": model},
        "e2e": {"value": round(value, 4), "unit": "Gflop/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def config_of(w, a, per_gpu=None):
    small = w["n"] * w["n"] * w["batch"] * 4 < (256 << 20)
    if per_gpu is None:
        per_gpu = -(-w["batch"] // max(1, a.gpus)) if w.get("global_batch") else w["batch"]
    return {"workload": w["desc"], "n": w["n"], "batch_per_gpu": per_gpu,
            "global_batch": w["batch"] if w.get("global_batch") else w["batch"] * a.gpus,
            "chunk": w["chunk"],
            "generator": w["kind"], "layout": "chunked interleaved" if w["chunk"] else "simple interleaved",
            "parallelism": f"batch split over {a.gpus} GPU(s), 1 all-reduce of the failure count",
            "l2": ("L2 flushed between steps (512 MB scratch write outside the per-step CUDA-event "
                   "pairs); step time = sum of per-step event durations" if small else
                   "inputs larger than L2 (126 MB); every step factors a distinct pre-generated buffer")}


# --------------------------------------------------------------------- clocks
class ClockSampler:
    """NVML SM-clock / clock-event-reason sampler.  The thread runs for the
    whole timed phase; only samples taken inside a marked window (the timed
    region, bracketed by mark_start/mark_stop) are reported."""

    def __init__(self, index):
        self.samples, self.reasons, self.max_mhz = [], 0, None
        self._all = []
        self._win = []
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self._rfn = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                pynvml.nvmlDeviceGetCurrentClocksThrottleReasons
        except Exception:
            self.nv = None

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                t = time.perf_counter()
                self._all.append((t, nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM),
                                  int(self._rfn(self.h))))
            except Exception:
                pass
            time.sleep(0.0002)

    def start(self):
        if self.nv is not None and self._t is None:
            self._stop.clear()
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
            time.sleep(0.002)

    def mark_start(self):
        self._win.append([time.perf_counter(), None])

    def mark_stop(self):
        if self._win:
            self._win[-1][1] = time.perf_counter()

    def sample_now(self, k=3):
        """Synchronous samples from the calling thread while queued kernels run
        (short timed regions can end before the sampler thread gets a turn)."""
        if self.nv is None:
            return
        for _ in range(k):
            try:
                self._all.append((time.perf_counter(), self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM),
                                  int(self._rfn(self.h))))
            except Exception:
                pass

    def stop(self):
        if self._t is not None:
            self._stop.set()
            self._t.join()
            self._t = None
        for t, mhz, r in self._all:
            if any(a <= t <= (b if b is not None else t) for a, b in self._win):
                self.samples.append(mhz)
                self.reasons |= r

    def report(self):
        names = [v for k, v in FLAG_NAMES.items() if self.reasons & k and k != 0x1]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(self.samples),
                "source": "NVML, sampled every ~0.2 ms inside the timed region"}


# --------------------------------------------------------------------- GPU side
def host_budget_bytes(local_world):
    """Per-rank cap on pinned host memory for the e2e leg: 40% of the host's
    available memory shared by the ranks of this node, at most 48 GiB."""
    avail = None
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("MemAvailable:"):
                avail = int(line.split()[1]) * 1024
    except OSError:
        pass
    if avail is None:
        avail = 64 << 30
    return int(min(48 << 30, 0.4 * avail / max(1, local_world)))


def median(xs):
    return statistics.median(xs) if xs else None


def per_n_sweep(bsp, torch, dev, stream, ns, batch, chunk, reps=5, conv=True, copy_ref_max_n=8,
                peak=6544.0, tag="1M"):
    """The "vs n" half of BASELINE's metric: every n in ``ns`` at ``batch``
    matrices (dd generator, chunk ``chunk``), the table's kernel, one launch
    per rep with the input regenerated and L2 flushed between reps (outside
    the event pair).  For n <= copy_ref_max_n a plain device copy of the same
    byte count is timed alongside (the small-n ceiling).  With ``conv`` the
    canonical path (canonical -> interleaved, factor, -> canonical) is timed
    too (BASELINE configs[3]), and for n <= CANON_MAX_N the fused canonical
    call (batch_spotrf_canonical: conversion inside the factorization kernel)."""
    maxn = max(ns)
    A = torch.empty(bsp.batch_interleaved_elems(maxn, batch, chunk), dtype=torch.float32, device=dev)
    canon = torch.empty(batch * maxn * maxn, dtype=torch.float32, device=dev) if conv else None
    info = torch.empty(batch, dtype=torch.int32, device=dev)
    cnt = torch.zeros(1, dtype=torch.int32, device=dev)
    flush = torch.empty((512 << 20) // 4, dtype=torch.float32, device=dev)
    Ev = lambda: torch.cuda.Event(enable_timing=True)
    rows = []
    for n in ns:
        elems = bsp.batch_interleaved_elems(n, batch, chunk)
        Av = A[:elems]
        t = bsp.bspotrf_get_tuning(n, chunk).as_dict()
        fact = []
        cnt.zero_()
        for _ in range(reps):
            bsp.bspotrf_synth_generate(n, batch, chunk, Av, kind="dd", seed=2017, stream=stream)
            bsp.bspotrf_fill_u32(flush, 0x3F800000, stream=stream)
            e0, e1 = Ev(), Ev()
            e0.record(stream)
            bsp.batch_spotrf_interleaved_ex(n, batch, chunk, Av, info, nfailed=cnt, stream=stream)
            e1.record(stream)
            fact.append((e0, e1))
        torch.cuda.synchronize(dev)
        if int(cnt.item()) != 0:
            raise SystemExit(f"bench per-n: {int(cnt.item())} failures on SPD input at n={n}")
        ms = median([x.elapsed_time(y) for x, y in fact])
        byt = batch * bytes_per_matrix(n)
        row = {"n": n, "variant": t["variant"], "ms": round(ms, 5),
               "gbs": round(byt / (ms * 1e-3) / 1e9, 1),
               "frac": round(byt / (ms * 1e-3) / 1e9 / peak, 4),
               "gflops": round(batch * flops_per_matrix(n) / (ms * 1e-3) / 1e9, 1)}
        if n <= copy_ref_max_n:
            half = byt // 2 // 4
            src = A[:half]
            dst = canon[:half] if canon is not None and canon.numel() >= half else torch.empty_like(src)
            cp = []
            for _ in range(reps):
                bsp.bspotrf_fill_u32(flush, 0x3F800000, stream=stream)
                e0, e1 = Ev(), Ev()
                e0.record(stream)
                dst.copy_(src)
                e1.record(stream)
                cp.append((e0, e1))
            torch.cuda.synchronize(dev)
            cms = median([x.elapsed_time(y) for x, y in cp])
            row["copy_gbs"] = round(byt / (cms * 1e-3) / 1e9, 1)
            row["vs_copy"] = round(cms / ms, 3)
        if conv:
            cv = canon[:batch * n * n]
            c_in, c_out = [], []
            for _ in range(max(2, reps - 2)):
                bsp.bspotrf_fill_u32(flush, 0x3F800000, stream=stream)
                e0, e1, e2 = Ev(), Ev(), Ev()
                e0.record(stream)
                bsp.batch_interleaved_to_canonical(n, batch, chunk, Av, cv, stream=stream)
                e1.record(stream)
                bsp.bspotrf_fill_u32(flush, 0x3F800000, stream=stream)
                e2.record(stream)
                e3 = Ev()
                bsp.batch_canonical_to_interleaved(n, batch, chunk, cv, Av, stream=stream)
                e3.record(stream)
                c_out.append((e0, e1))
                c_in.append((e2, e3))
            torch.cuda.synchronize(dev)
            mi = median([x.elapsed_time(y) for x, y in c_in])
            mo = median([x.elapsed_time(y) for x, y in c_out])
            cb = batch * 8 * n * n
            row["convert_in_gbs"] = round(cb / (mi * 1e-3) / 1e9, 1)
            row["convert_out_gbs"] = round(cb / (mo * 1e-3) / 1e9, 1)
            row["canonical_path_gflops"] = round(batch * flops_per_matrix(n) / ((mi + ms + mo) * 1e-3) / 1e9, 1)
            if n <= bsp.CANON_MAX_N:
                # the fused canonical call (batch_spotrf_canonical) on the same
                # matrices in canonical storage: algorithmic bytes as above
                fz = []
                cnt.zero_()
                for _ in range(reps):
                    bsp.bspotrf_synth_generate(n, batch, chunk, Av, kind="dd", seed=2017, stream=stream)
                    bsp.batch_interleaved_to_canonical(n, batch, chunk, Av, cv, stream=stream)
                    bsp.bspotrf_fill_u32(flush, 0x3F800000, stream=stream)
                    e0, e1 = Ev(), Ev()
                    e0.record(stream)
                    bsp.batch_spotrf_canonical(n, batch, cv, info, nfailed=cnt, stream=stream)
                    e1.record(stream)
                    fz.append((e0, e1))
                torch.cuda.synchronize(dev)
                if int(cnt.item()) != 0:
                    raise SystemExit(f"bench per-n: {int(cnt.item())} canonical failures on SPD input at n={n}")
                mf = median([x.elapsed_time(y) for x, y in fz])
                row["canonical_fused_gbs"] = round(byt / (mf * 1e-3) / 1e9, 1)
                row["canonical_fused_gflops"] = round(batch * flops_per_matrix(n) / (mf * 1e-3) / 1e9, 1)
        rows.append(row)
    del A, canon, flush
    torch.cuda.empty_cache()
    return {"batch": batch, "chunk": chunk, "generator": "dd", "reps": reps, "peak_gbs": peak,
            "timing": "median of per-launch CUDA-event times; input regenerated and L2 flushed "
                      "(512 MB write) before every launch, outside the event pair",
            "rows": rows, "tag": tag}


def run_ours(a, w):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_gatesklpd17_b200 as bsp
    from paper_conf_ipps_gatesklpd17_b200 import multi_gpu

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", str(world)))
    gpu = 0 if a.same_device else local
    torch.cuda.set_device(gpu)
    dev = torch.device("cuda", gpu)
    if world > 1:
        if a.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:                                  # test mode: several ranks may share one GPU
            dist.init_process_group("gloo")
    bsp.lib()

    n, chunk, kind = w["n"], w["chunk"], w["kind"]
    fail_period = w.get("fail_period", 0)
    # One global batch of independent matrices, cut into chunk-aligned slices of
    # GLOBAL indices (multi_gpu.rank_slice).  Strong scaling (c5): the global batch
    # is fixed; weak scaling: it is the per-GPU batch times the world size.
    Bg = w["batch"] if w.get("global_batch") else w["batch"] * world
    mk = lambda: multi_gpu.RankBatch(n, Bg, chunk, kind=kind, seed=2017, fail_seed=2018,
                                     fail_period=fail_period, device=dev)
    first = mk()
    B, b0 = first.count, first.b0
    tune = json.loads(a.tune) if a.tune else None
    tsel = bsp.bspotrf_get_tuning(n, chunk).as_dict() if tune is None else tune
    elems = bsp.batch_interleaved_elems(n, B, chunk) if B else 0
    buf_bytes = max(elems, 4) * 4 + max(B, 1) * 4
    free, _ = torch.cuda.mem_get_info(dev)
    fit = int(min(a.max_pool_gb * 2**30, 0.80 * free) // buf_bytes)
    P = max(1, min(a.steps, fit))
    P = multi_gpu.min_over_ranks(P, device=dev)        # same pool size -> same collectives
    stream = torch.cuda.current_stream(dev)
    pool = [first] + [mk() for _ in range(P - 1)]

    def regen():
        for rb in pool:
            rb.regenerate(stream=stream)
            rb.nfailed.zero_()

    def barrier():
        if world > 1:
            dist.barrier()

    def step(i):
        rb = pool[i % P]
        rb.factor(stream=stream, tune=tune, reset=False)
        rb.reduce_failures()                   # a9: the one collective, 4 bytes (N > 1)

    regen()
    for i in range(a.warmup):
        step(i)
    torch.cuda.synchronize(dev)
    regen()
    torch.cuda.synchronize(dev)

    # L2 hygiene: a step's input larger than L2 needs nothing (every step also
    # factors a distinct buffer); a smaller one gets an L2 flush (a 512 MB
    # scratch write) between steps, OUTSIDE the per-step event pairs, and the
    # step time is the sum of the per-step event durations.
    small = elems * 4 < (256 << 20)
    flush = torch.empty((512 << 20) // 4, dtype=torch.float32, device=dev) if small else None
    clk = ClockSampler(gpu)
    clk.start()
    total_ms, launch_ms, done = 0.0, [], 0
    fails = 0
    while done < a.steps:
        g = min(P, a.steps - done)
        if done > 0:
            regen()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(g)]
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        torch.cuda.synchronize(dev)
        clk.mark_start()
        e0.record(stream)
        for i in range(g):
            if small:
                bsp.bspotrf_fill_u32(flush, 0x3F800000, stream=stream)
            ev[i][0].record(stream)
            step(i)
            ev[i][1].record(stream)
        e1.record(stream)
        clk.sample_now(1)                      # the queued steps are running now
        torch.cuda.synchronize(dev)
        clk.mark_stop()
        barrier()
        steps_ms = [s.elapsed_time(t) for s, t in ev]
        total_ms += sum(steps_ms) if small else e0.elapsed_time(e1)
        launch_ms += steps_ms
        fails += sum(int(pool[i].nfailed.item()) for i in range(g))   # global (all-reduced) counts
        done += g
    total_ms, mean_launch_ms = multi_gpu.max_over_ranks([total_ms, statistics.mean(launch_ms)], device=dev)
    clk.stop()
    # correctness guard on the timed output: SPD input -> no failure; injected
    # failures -> the global count equals the enumerated plan (pin P10)
    expect = 0
    if fail_period:
        import synth
        expect = synth.expected_fail_count(n, 2018, fail_period, 0, Bg)
    last = min(P, a.steps)
    bad = sum(int((pool[i].info[:B] != 0).sum().item()) for i in range(last))
    if (not fail_period and bad) or fails != expect * a.steps:
        raise SystemExit(f"bench: {bad} nonzero info / {fails} counted failures, expected "
                         f"{expect} per step")

    ms_per_step = total_ms / a.steps
    value = multi_gpu.job_throughput(B, world, ms_per_step, flops_per_matrix(n), global_units=Bg)
    alg_bytes = B * bytes_per_matrix(n)
    achieved = alg_bytes / (mean_launch_ms * 1e-3) / 1e9
    peak, peak_src = measured_peak()
    hbm_gbs = Bg * bytes_per_matrix(n) / (ms_per_step * 1e-3) / 1e9

    # ---------------- e2e: the host-buffer C-ABI call, copies inside the timed region
    e2e = None
    del pool, first
    torch.cuda.empty_cache()
    if not a.no_e2e and a.e2e_steps > 0:
        e2e = run_e2e(a, bsp, torch, dist, dev, stream, world, local_world, n, B, b0, chunk, kind,
                      fail_period, barrier)

    per_n = per_n_large = None
    if world == 1 and a.per_n != "none":
        ns = parse_ns(a.per_n)
        per_n = per_n_sweep(bsp, torch, dev, stream, ns, 1 << 20, 32, peak=peak, tag="1M")
        small_ns = [x for x in ns if x <= 8]
        if small_ns:
            per_n_large = per_n_sweep(bsp, torch, dev, stream, small_ns, 1 << 26, 32, conv=True,
                                      peak=peak, tag="64M (n <= 8: out of the launch-latency regime)")

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_oracle_rate(n, kind, a.cpu_seconds, B)
        t1 = cpu_oracle_rate(n, kind, a.cpu_seconds / 2, B, cores=1)
        cpu["t1"] = {"value": t1["value"], "unit": t1["unit"], "cores": 1, "sample": t1["sample"]}
        cpu["cpu_model"] = cpu_model()
        cpu["host_cores"] = host_cores()

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": "Gflop/s", "n_gpus": world,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(ms_per_step, 5),
        "higher_is_better": True, "scaling": "strong" if w.get("global_batch") else "weak",
        "vs_baseline": None, "dtype": "f32",
        "data": "synthetic (seeded counter-hash generator on device)",
        "config": dict(config_of(w, a, per_gpu=B), tuning=tsel),
        "hbm_gbs": round(hbm_gbs, 2),
        "roofline": {"bound": "hbm", "achieved": round(achieved, 2), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "traffic": traffic_from_profiles(w),
                     "peak_source": peak_src,
                     "kernel": f"factorization kernel (variant {tsel['variant']}), "
                               f"{bytes_per_matrix(n)} B/matrix x {B} matrices per launch, "
                               f"mean launch {mean_launch_ms:.4f} ms"},
        "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": a.steps,
        "clocks": clk.report(),
        "per_n": per_n, "per_n_large_batch": per_n_large,
    }
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def parse_ns(spec):
    out = []
    for part in spec.split(","):
        if "-" in part:
            lo, hi = part.split("-")
            out += list(range(int(lo), int(hi) + 1))
        elif part:
            out.append(int(part))
    return out


def run_e2e(a, bsp, torch, dist, dev, stream, world, local_world, n, B, b0, chunk, kind,
            fail_period, barrier):
    """e2e: the public host-buffer call (batch_spotrf_interleaved_host) on pinned
    host storage, host<->device traffic inside the timed region.  The pinned
    buffer is capped per rank (host_budget_bytes); a rank slice larger than the
    cap is measured on its leading chunk-aligned part, stated in "sample"."""
    cap = host_budget_bytes(local_world)
    C = chunk if chunk > 0 else 32
    Be = B
    while Be > C and bsp.batch_interleaved_elems(n, Be, chunk) * 4 > cap:
        Be = max(C, (Be // 2) // C * C)
    Be = multi_gpu_min(Be, dev, dist, world)
    elems = bsp.batch_interleaved_elems(n, Be, chunk)
    dA = torch.empty(elems, dtype=torch.float32, device=dev)      # pristine input, on device
    bsp.bspotrf_synth_generate(n, Be, chunk, dA, kind=kind, seed=2017, b0=b0,
                               fail_seed=2018, fail_period=fail_period, stream=stream)
    torch.cuda.synchronize(dev)
    hA = torch.empty(elems, dtype=torch.float32).pin_memory()
    hinfo = torch.empty(Be, dtype=torch.int32).pin_memory()
    expect = 0
    if fail_period:
        import synth
        expect = synth.expected_fail_count(n, 2018, fail_period, 0, Be * world) if world == 1 else None

    def e2e_run(slab):
        times = []
        for s in range(a.e2e_steps + 1):
            hA.copy_(dA)                       # restore the input (outside the timed region)
            torch.cuda.synchronize(dev)
            barrier()
            t0 = time.perf_counter()
            nf = bsp.batch_spotrf_interleaved_host(n, Be, chunk, hA, hinfo, slab=slab, stream=stream)
            if world > 1:
                c = torch.tensor([nf], dtype=torch.int32, device=dev)
                dist.all_reduce(c)
                nf = int(c.item())
            dt = time.perf_counter() - t0
            if expect is not None and nf != expect:
                raise SystemExit(f"bench e2e: {nf} failures, expected {expect}")
            if s > 0:                          # first call warms the pool / streams
                times.append(dt)
        tt = torch.tensor([sum(times) / len(times)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        return float(tt.item())

    hb = bsp.batch_spotrf_host_bytes(n, Be, chunk)
    t_zero = e2e_run(0)                         # zero-copy on pinned buffers
    slab = max(C, ((32 << 20) // (2 * n * (n + 1))) // C * C)
    t_pipe = e2e_run(slab)                      # the copy pipeline
    Btot = Be * world
    gfl = lambda t: round(Btot * flops_per_matrix(n) / t / 1e9, 3)
    paths = {"zero_copy": {"value": gfl(t_zero), "ms_per_step": round(t_zero * 1e3, 3), "slab": 0,
                           "path": "batch_spotrf_interleaved_host(slab=0) on pinned host interleaved "
                                   "storage: zero-copy, the factorization kernel reads/writes host "
                                   "memory over PCIe"},
             "copy_pipeline": {"value": gfl(t_pipe), "ms_per_step": round(t_pipe * 1e3, 3),
                               "slab": slab,
                               "path": f"batch_spotrf_interleaved_host(slab={slab}): 3-stream slab "
                                       "pipeline, lower-triangle 2-D copies H2D / kernel / D2H"}}
    best = "zero_copy" if t_zero <= t_pipe else "copy_pipeline"
    tb = min(t_zero, t_pipe)
    out = {"value": gfl(tb), "unit": "Gflop/s", "h2d_bytes_per_step": hb,
           "d2h_bytes_per_step": hb + 4 * Be + 4, "ms_per_step": round(tb * 1e3, 3),
           "path": paths[best]["path"], "pcie_gbs_each_way": round(hb / tb / 1e9, 2),
           "paths": paths}
    if Be != B:
        out["sample"] = (f"leading {Be} of the rank's {B} matrices per rank (pinned host buffer "
                         f"capped at {cap / 2**30:.1f} GiB per rank)")
    del dA, hA, hinfo
    torch.cuda.empty_cache()
    return out


def multi_gpu_min(v, dev, dist, world):
    if world == 1:
        return v
    from paper_conf_ipps_gatesklpd17_b200 import multi_gpu
    return multi_gpu.min_over_ranks(v, device=dev)


def main():
    sys.setswitchinterval(0.0002)   # let the NVML clock sampler run during the timed region
    a = parse()
    w = workload(a)
    if a.impl == "reference":
        return run_reference(a, w)
    return run_ours(a, w)


if __name__ == "__main__":
    sys.exit(main())
