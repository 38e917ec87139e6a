"""GPU: batch_spotrf_canonical (factorization on canonical storage, layout
conversion fused; include/bspotrf.h) against the FP64 oracle, which works on
canonical column-major matrices natively, and bitwise against the interleaved
path (convert -> table kernel -> convert back) on the same matrices (pin P8:
same per-element FP32 op sequence)."""
import numpy as np
import pytest

import oracle
import synth
from oracle import checks

import paper_conf_ipps_gatesklpd17_b200 as bsp
from gpu_helpers import torch_mod

pytestmark = pytest.mark.gpu


def _run_canon(n, canon, with_count=True):
    torch = torch_mod()
    batch = canon.shape[0]
    dA = torch.from_numpy(canon.reshape(-1).copy()).cuda()
    dinfo = torch.full((max(batch, 1),), -7, dtype=torch.int32, device="cuda")
    dcnt = torch.zeros(1, dtype=torch.int32, device="cuda") if with_count else None
    bsp.batch_spotrf_canonical(n, batch, dA, dinfo, nfailed=dcnt)
    torch.cuda.synchronize()
    out = dA.cpu().numpy().reshape(batch, n * n)
    return out, dinfo.cpu().numpy()[:batch], (int(dcnt.item()) if with_count else None)


def _check(n, canon, out, info, cnt):
    L64, info64 = oracle.potrf(n, canon)
    r = checks.accept(n, canon, out, info, L64, info64)
    bad = np.nonzero(~r["ok"])[0]
    assert bad.size == 0, f"n={n}: {bad.size} matrices fail, first {bad[:5]}"
    assert r["strict"].max() <= checks.STRICT_TOL
    # the strict upper triangle (NaN sentinels in these inputs) is never read
    # (a read would poison L) nor written
    assert checks.upper_bits_unchanged(n, canon, out).all()
    if cnt is not None:
        assert cnt == int((info64 != 0).sum())
    return info64


@pytest.mark.parametrize("n", list(range(1, bsp.CANON_MAX_N + 1)))
@pytest.mark.parametrize("batch", [1, 31, 4096 + 32 * 3 + 17])
def test_canonical_matches_oracle(n, batch):
    b = np.arange(batch, dtype=np.uint64)
    canon = synth.generate(n, "dd", 2017, b, upper="nan", fail_seed=2018, fail_period=53)
    out, info, cnt = _run_canon(n, canon)
    _check(n, canon, out, info, cnt)


@pytest.mark.parametrize("n", [2, 7, 12, 16, 19, 20])
@pytest.mark.parametrize("kind", ["als", "l0"])
def test_canonical_generators(n, kind):
    batch = 3000 + 5
    b = np.arange(batch, dtype=np.uint64)
    canon = synth.generate(n, kind, 11, b, upper="nan", fail_seed=12, fail_period=97)
    out, info, cnt = _run_canon(n, canon)
    info64 = _check(n, canon, out, info, cnt)
    if kind == "l0":                          # pin P2: exactly L0 where info = 0
        L0 = synth.l0_factor(n, 11, b)
        ok = info64 == 0
        low = np.tril(np.ones((n, n), bool)).T.reshape(-1)
        L0c = L0.transpose(0, 2, 1).reshape(batch, n * n)      # column-major flat (i + j*n)
        assert np.array_equal(out[ok][:, low], L0c[ok][:, low])


@pytest.mark.parametrize("n", [3, 8, 13, 16, 20])
def test_canonical_bitwise_equals_interleaved_path(n):
    """Fused canonical call == canonical -> interleaved -> table kernel ->
    canonical, bit for bit (L and info), failures included."""
    torch = torch_mod()
    batch = 8192 + 77
    b = np.arange(batch, dtype=np.uint64)
    canon = synth.generate(n, "als", 5, b, upper="mirror", fail_seed=6, fail_period=31)
    out, info, _ = _run_canon(n, canon, with_count=False)
    src = torch.from_numpy(canon.reshape(-1).copy()).cuda()
    inter = torch.zeros(bsp.batch_interleaved_elems(n, batch, 32), device="cuda")
    bsp.batch_canonical_to_interleaved(n, batch, 32, src, inter)
    dinfo = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bsp.batch_spotrf_interleaved(n, batch, 32, inter, dinfo)
    back = torch.zeros(batch * n * n, device="cuda")
    bsp.batch_interleaved_to_canonical(n, batch, 32, inter, back)
    torch.cuda.synchronize()
    ref = back.cpu().numpy().reshape(batch, n * n)
    assert np.array_equal(info, dinfo.cpu().numpy())
    low = np.tril(np.ones((n, n), bool)).T.reshape(-1)
    ok = info == 0                            # failed matrices: only final columns are defined
    assert np.array_equal(out.view(np.uint32)[ok][:, low], ref.view(np.uint32)[ok][:, low])
    # the strict upper (mirrored input) is bitwise the input
    assert np.array_equal(out.view(np.uint32)[:, ~low], canon.view(np.uint32)[:, ~low])


@pytest.mark.parametrize("n", [4, 16, 20])
def test_canonical_large_batch_sampled(n):
    """1M matrices (4 KiB-32 KiB canonical groups over every SM many times):
    the fused count equals the enumerated failure plan; sampled matrices match
    the oracle; the upper triangle of sampled matrices is untouched."""
    torch = torch_mod()
    batch = 1 << 20
    period = 1009
    dA = torch.empty(batch * n * n, device="cuda")
    # canonical input from the device generator: interleaved (chunk 32), then
    # converted (both pinned elsewhere against the host generator / layout)
    inter = torch.empty(bsp.batch_interleaved_elems(n, batch, 32), device="cuda")
    bsp.bspotrf_synth_generate(n, batch, 32, inter, kind="dd", seed=2017, upper="nan",
                               fail_seed=2018, fail_period=period)
    bsp.batch_interleaved_to_canonical(n, batch, 32, inter, dA)
    del inter
    dinfo = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    dcnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    bsp.batch_spotrf_canonical(n, batch, dA, dinfo, nfailed=dcnt)
    torch.cuda.synchronize()
    assert int(dcnt.item()) == synth.expected_fail_count(n, 2018, period, 0, batch)
    rng = np.random.default_rng(n)
    idx = np.unique(np.concatenate([rng.choice(batch, 3000, replace=False), [0, 31, 32, batch - 1]]))
    canon = synth.generate(n, "dd", 2017, idx.astype(np.uint64), upper="nan", fail_seed=2018,
                           fail_period=period)
    out = dA.view(batch, n * n)[torch.from_numpy(idx).cuda()].cpu().numpy()
    info = dinfo[torch.from_numpy(idx).cuda()].cpu().numpy()
    _check(n, canon, out, info, None)
