"""Helpers for the GPU parity tests (test infrastructure).

Inputs are generated on the HOST by synth/ (seeded), laid out by the oracle's
layout definition, uploaded, factored by the CUDA path through the C ABI, and
compared with the FP64 oracle on the same inputs.
"""
import numpy as np

import oracle
import synth
from oracle import checks, layout

import paper_conf_ipps_gatesklpd17_b200 as bsp


def torch_mod():
    import torch
    return torch


def make_batch(n, batch, chunk, kind="dd", seed=2017, upper="nan", fail_seed=0, fail_period=0,
               b0=0):
    """Host canonical batch + its interleaved storage with sentinel pad lanes."""
    b = np.arange(b0, b0 + batch, dtype=np.uint64)
    canon = synth.generate(n, kind, seed, b, upper=upper, fail_seed=fail_seed,
                           fail_period=fail_period)
    inter = layout.to_interleaved(n, chunk, canon, fill_bits=synth.PAD_BITS)
    return canon, inter


def run_gpu(n, batch, chunk, inter, tune=None, with_count=True):
    torch = torch_mod()
    dA = torch.from_numpy(inter.copy()).cuda()
    dinfo = torch.full((max(batch, 1),), -7, dtype=torch.int32, device="cuda")
    dcnt = torch.zeros(1, dtype=torch.int32, device="cuda") if with_count else None
    bsp.batch_spotrf_interleaved_ex(n, batch, chunk, dA, dinfo, nfailed=dcnt, tune=tune)
    torch.cuda.synchronize()
    out = dA.cpu().numpy()
    info = dinfo.cpu().numpy()[:batch]
    cnt = int(dcnt.item()) if with_count else None
    return out, info, cnt


def assert_parity(n, batch, chunk, canon, inter_in, inter_out, info, cnt=None, emulate=True):
    """O1-O4 against the FP64 oracle, plus pad lanes and (P8) bitwise equality
    with the Fig. 9 FP32 op-order emulator."""
    L64, info64 = oracle.potrf(n, canon)
    got = layout.from_interleaved(n, batch, chunk, inter_out)
    r = checks.accept(n, canon, got, info, L64, info64)
    bad = np.nonzero(~r["ok"])[0]
    assert bad.size == 0, (
        f"n={n} batch={batch} chunk={chunk}: {bad.size} matrices fail; first {bad[:5]} "
        f"info {info[bad[:5]]} vs {info64[bad[:5]]}, err {r['err'][bad[:5]]}, resid {r['resid'][bad[:5]]}")
    # R10 diagnostic: the literal 1e-4 on entries >= 1e-2 x column max
    # (fast-math REGX, reading R4, is held to 10x: approximate sqrt/rcp)
    stol = checks.STRICT_TOL if emulate else 10 * checks.STRICT_TOL
    assert r["strict"].max() <= stol, f"strict relative error {r['strict'].max():.3e}"
    # O4: strict upper triangle and pad lanes bitwise untouched
    assert checks.upper_bits_unchanged(n, canon, got).all()
    pads = layout.pad_lane_offsets(n, batch, chunk)
    assert np.array_equal(inter_out.view(np.uint32)[pads], inter_in.view(np.uint32)[pads])
    if cnt is not None:
        assert cnt == int((info64 != 0).sum())
    if emulate:
        W, infoe = oracle.spotrf_fig9_fp32(n, canon)
        assert np.array_equal(infoe, info)
        ok = info == 0
        low = np.tril(np.ones((n, n), bool)).T.reshape(-1)   # canonical flat lower mask
        gb = got.view(np.uint32)[ok][:, low]
        wb = W.view(np.uint32)[ok][:, low]
        mism = np.nonzero((gb != wb).any(axis=1))[0]
        assert mism.size == 0, f"{mism.size} SPD matrices differ bitwise from the Fig.9 emulator"
    return r
