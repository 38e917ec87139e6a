"""GPU parity at BASELINE.json's full sizes, in the launch configuration
bench.py times (tuning table, device generator), checked on sampled matrices
the oracle recomputes one by one, plus properties that hold at any size."""
import numpy as np
import pytest

import oracle
import synth
from oracle import checks, layout

import paper_conf_ipps_gatesklpd17_b200 as bsp
from gpu_helpers import torch_mod

pytestmark = pytest.mark.gpu


def gather(dA, n, batch, chunk, b_idx):
    """Canonical (len(b), n*n) view of sampled matrices from device storage."""
    torch = torch_mod()
    e = np.arange(n * n)
    offs = layout.offset(n, batch, chunk, b_idx[:, None], (e % n)[None, :], (e // n)[None, :])
    t = torch.from_numpy(offs.reshape(-1).astype(np.int64)).to(dA.device)
    return torch.take(dA, t).cpu().numpy().reshape(len(b_idx), n * n)


def sample_idx(batch, k=4096, seed=0):
    rng = np.random.default_rng(seed)
    s = rng.choice(batch, size=min(k, batch), replace=False)
    edge = np.r_[np.arange(min(512, batch)), np.arange(max(0, batch - 512), batch)]
    return np.unique(np.r_[s, edge]).astype(np.int64)


def factor_sampled(n, batch, chunk, kind, seed=2017, fail_period=0, upper="nan"):
    torch = torch_mod()
    dA = torch.empty(bsp.batch_interleaved_elems(n, batch, chunk), dtype=torch.float32, device="cuda")
    bsp.bspotrf_synth_generate(n, batch, chunk, dA, kind=kind, seed=seed, upper=upper,
                               fail_seed=2018, fail_period=fail_period)
    info = torch.empty(batch, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    bsp.batch_spotrf_interleaved_ex(n, batch, chunk, dA, info, nfailed=cnt)
    torch.cuda.synchronize()
    return dA, info, cnt


def check_sample(n, batch, chunk, kind, dA, info, seed=2017, fail_period=0, upper="nan"):
    b = sample_idx(batch)
    A = synth.generate(n, kind, seed, b.astype(np.uint64), upper=upper, fail_seed=2018,
                       fail_period=fail_period)
    L64, info64 = oracle.potrf(n, A)
    got = gather(dA, n, batch, chunk, b)
    ginfo = info.cpu().numpy()[b]
    r = checks.accept(n, A, got, ginfo, L64, info64)
    assert r["ok"].all(), np.nonzero(~r["ok"])[0][:10]
    assert r["strict"].max() <= checks.STRICT_TOL
    assert checks.upper_bits_unchanged(n, A, got).all()
    return got, b


def test_c1_n8_b16384_chunk32_full_check():
    n, batch, chunk = 8, 16384, 32
    dA, info, cnt = factor_sampled(n, batch, chunk, "dd")
    b = np.arange(batch)
    A = synth.generate(n, "dd", 2017, b.astype(np.uint64), upper="nan")
    L64, info64 = oracle.potrf(n, A)
    got = layout.from_interleaved(n, batch, chunk, dA.cpu().numpy())
    r = checks.accept(n, A, got, info.cpu().numpy(), L64, info64)
    assert r["ok"].all() and int(cnt.item()) == 0
    assert r["err"].max() < 1e-5 and r["resid"].max() < 2.0


@pytest.mark.parametrize("chunk", [32, 0, 64, 128])
def test_c2_n16_b1m(chunk):
    n, batch = 16, 1 << 20
    dA, info, cnt = factor_sampled(n, batch, chunk, "dd")
    assert int(cnt.item()) == 0 and int((info != 0).sum().item()) == 0
    got, b = check_sample(n, batch, chunk, "dd", dA, info)
    if chunk != 32:     # P8 across layouts on the same sampled matrices
        dA32, _, _ = factor_sampled(n, batch, 32, "dd")
        ref = gather(dA32, n, batch, 32, b)
        assert np.array_equal(ref.view(np.uint32), got.view(np.uint32))


def test_c3_n32_b4m_als():
    n, batch, chunk = 32, 1 << 22, 32
    dA, info, cnt = factor_sampled(n, batch, chunk, "als")
    assert int(cnt.item()) == 0
    check_sample(n, batch, chunk, "als", dA, info)


@pytest.mark.parametrize("n", [1, 4, 24, 33, 48, 64])
def test_c4_nsweep_b1m(n):
    batch, chunk = 1 << 20, 32
    dA, info, cnt = factor_sampled(n, batch, chunk, "dd", fail_period=1009)
    exp = synth.expected_fail_count(n, 2018, 1009, 0, batch)
    assert int(cnt.item()) == exp == int((info != 0).sum().item())
    check_sample(n, batch, chunk, "dd", dA, info, fail_period=1009)


def test_c5_partitioned_fail_count_on_one_gpu():
    """C5's partition (chunk-aligned global slices per rank) run rank by rank
    on one GPU: the summed count equals the enumerated global count (P10)."""
    from paper_conf_ipps_gatesklpd17_b200 import multi_gpu
    torch = torch_mod()
    n, B, chunk, P = 32, 1 << 21, 32, 1009
    total = 0
    for world in (1, 2, 8):
        total = 0
        for rank in range(world):
            b0, cnt = multi_gpu.rank_slice(B, world, rank, chunk)
            dA = torch.empty(bsp.batch_interleaved_elems(n, cnt, chunk), device="cuda")
            bsp.bspotrf_synth_generate(n, cnt, chunk, dA, kind="dd", seed=2017, b0=b0,
                                       fail_seed=2018, fail_period=P)
            info = torch.empty(cnt, dtype=torch.int32, device="cuda")
            c = torch.zeros(1, dtype=torch.int32, device="cuda")
            bsp.batch_spotrf_interleaved_ex(n, cnt, chunk, dA, info, nfailed=c)
            total += int(c.item())
        assert total == synth.expected_fail_count(n, 2018, P, 0, B)
