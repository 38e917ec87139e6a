"""GPU: layout conversion kernels, the device generator, and the host-buffer
end-to-end call -- all through the C ABI, against the oracle / synth."""
import numpy as np
import pytest

import synth
from oracle import layout

import paper_conf_ipps_gatesklpd17_b200 as bsp
from gpu_helpers import assert_parity, make_batch, run_gpu, torch_mod

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 12, 14, 16, 31, 32, 33, 45, 50, 63, 64])
@pytest.mark.parametrize("chunk", [32, 64, 0, 160])
@pytest.mark.parametrize("batch", [517, 1024, 96, 1, 1184, 1002])
def test_conversion_matches_layout_definition(n, chunk, batch):
    """The v2 kernel (128-bit on both sides) takes every full 32-matrix group
    when C % 4 == 0: n <= 5 as whole-group blocks (path A, several groups per
    tile, a partial last block at batch 1184 = 37 groups), n >= 6 as balanced
    element slices with aligned float4 slots (path B; odd n: phase != 0, edge
    slots stored by scalars).  The v1 kernel takes the ragged last group
    (batch 517, 1002) and chunk 0 with batch % 4 != 0 (1002: 32-bit
    interleaved accesses); batch 1: v1 only."""
    torch = torch_mod()
    rng = np.random.default_rng(n * 1000 + chunk)
    canon = rng.standard_normal((batch, n * n)).astype(np.float32)
    expect = layout.to_interleaved(n, chunk, canon, fill_bits=synth.PAD_BITS)
    dsrc = torch.from_numpy(canon).cuda()
    ddst = torch.zeros(expect.size, dtype=torch.float32, device="cuda")
    bsp.bspotrf_fill_u32(ddst, synth.PAD_BITS)
    bsp.batch_canonical_to_interleaved(n, batch, chunk, dsrc, ddst)
    got = ddst.cpu().numpy()
    assert np.array_equal(got.view(np.uint32), expect.view(np.uint32))   # incl. pads untouched
    back = torch.full((batch * n * n,), 7.0, device="cuda")
    bsp.batch_interleaved_to_canonical(n, batch, chunk, ddst, back)
    assert np.array_equal(back.cpu().numpy().view(np.uint32), canon.reshape(-1).view(np.uint32))


def _roundtrip_exact(n, batch, chunk, seed):
    torch = torch_mod()
    rng = np.random.default_rng(seed)
    canon = rng.standard_normal((batch, n * n), dtype=np.float32)
    expect = layout.to_interleaved(n, chunk, canon, fill_bits=synth.PAD_BITS)
    dsrc = torch.from_numpy(canon).cuda()
    ddst = torch.zeros(expect.size, dtype=torch.float32, device="cuda")
    bsp.bspotrf_fill_u32(ddst, synth.PAD_BITS)
    bsp.batch_canonical_to_interleaved(n, batch, chunk, dsrc, ddst)
    assert np.array_equal(ddst.cpu().numpy().view(np.uint32), expect.view(np.uint32))
    back = torch.full((batch * n * n,), 7.0, device="cuda")
    bsp.batch_interleaved_to_canonical(n, batch, chunk, ddst, back)
    assert np.array_equal(back.cpu().numpy().view(np.uint32), canon.reshape(-1).view(np.uint32))


@pytest.mark.parametrize("path", ["v4", "v3", "v2"])
@pytest.mark.parametrize("n", [6, 7, 10, 11, 12, 14, 17, 18, 30, 33, 34, 50, 61, 62, 64])
@pytest.mark.parametrize("chunk,batch", [(32, 1184), (0, 9632), (96, 4096 + 32 * 7 + 5)])
def test_conversion_paths_forced(monkeypatch, path, n, chunk, batch):
    """v4 (odd n: whole-group image + one bulk store), v3 (fixed 32-element
    slices, per-lane constant row phases, carries between
    slices) and v2 (proportional / aligned slices), each forced on every n
    class -- E % 4 in {0, 1}, E % 8 in {0, 4}, the last slice 1..32 wide -- with
    small group counts, where every group is cut into many segments (a unit =
    a few slices: partial first / last slots stored by scalars)."""
    monkeypatch.setenv("BSPOTRF_CONVERT_PATH", path)
    _roundtrip_exact(n, batch, chunk, seed=n * 7 + chunk)


@pytest.mark.parametrize("n,batch", [(7, 1 << 21), (10, 1 << 20), (63, 1 << 16), (62, 3 * 1 << 15)])
def test_conversion_large_batch(n, batch):
    """Default paths at batches where v3 runs one or two segments per group
    (whole-row streams with carries across every slice) and every persistent
    warp loops over many units."""
    _roundtrip_exact(n, batch, 32, seed=n)


@pytest.mark.parametrize("kind", ["dd", "als", "l0"])
@pytest.mark.parametrize("n", [1, 2, 7, 16, 32, 64])
@pytest.mark.parametrize("upper", ["mirror", "nan", "keep"])
def test_device_generator_matches_host(kind, n, upper):
    torch = torch_mod()
    batch, chunk, b0 = 300, 32, 12345
    dA = torch.zeros(bsp.batch_interleaved_elems(n, batch, chunk), dtype=torch.float32, device="cuda")
    bsp.bspotrf_fill_u32(dA, synth.PAD_BITS)
    bsp.bspotrf_synth_generate(n, batch, chunk, dA, kind=kind, seed=2017, b0=b0, upper=upper,
                               fail_seed=2018, fail_period=11)
    got = dA.cpu().numpy()
    host = synth.generate(n, kind, 2017, np.arange(b0, b0 + batch, dtype=np.uint64),
                          upper="nan" if upper == "nan" else "mirror", fail_seed=2018, fail_period=11)
    expect = layout.to_interleaved(n, chunk, host, fill_bits=synth.PAD_BITS)
    if upper == "keep":
        # strict upper not written: it still holds the fill pattern
        canon_exp = host.copy()
        su = np.triu(np.ones((n, n), bool), 1).T.reshape(-1)   # canonical flat strict upper
        canon_exp.view(np.uint32)[:, su] = synth.PAD_BITS
        expect = layout.to_interleaved(n, chunk, canon_exp, fill_bits=synth.PAD_BITS)
    assert np.array_equal(got.view(np.uint32), expect.view(np.uint32))


def test_generator_partition_invariance_chunk0():
    torch = torch_mod()
    n, batch = 9, 1000
    full = torch.zeros(batch * n * n, device="cuda")
    bsp.bspotrf_synth_generate(n, batch, 0, full, kind="als", seed=3)
    parts = []
    for b0 in range(0, batch, 250):
        p = torch.zeros(250 * n * n, device="cuda")
        bsp.bspotrf_synth_generate(n, 250, 0, p, kind="als", seed=3, b0=b0)
        parts.append(layout.from_interleaved(n, 250, 0, p.cpu().numpy()))
    a = layout.from_interleaved(n, batch, 0, full.cpu().numpy())
    assert np.array_equal(a.view(np.uint32), np.concatenate(parts).view(np.uint32))


@pytest.mark.parametrize("n,chunk,slab", [(8, 32, 0), (16, 32, 4096), (16, 64, 3 * 64),
                                          (21, 32, 1024), (32, 32, 2048), (5, 0, 500), (40, 0, 0),
                                          (12, 128, 256), (48, 32, 1024), (64, 64, 640)])
def test_host_end_to_end(n, chunk, slab):
    torch = torch_mod()
    batch = 5000 + 13
    canon, inter = make_batch(n, batch, chunk, kind="dd", fail_seed=1, fail_period=97)
    hA = torch.from_numpy(inter.copy()).pin_memory()
    hinfo = torch.full((batch,), -9, dtype=torch.int32).pin_memory()
    nf = bsp.batch_spotrf_interleaved_host(n, batch, chunk, hA, hinfo, slab=slab)
    out = hA.numpy()
    info = hinfo.numpy()
    assert nf == int((info != 0).sum())
    assert_parity(n, batch, chunk, canon, inter, out, info, nf)
    # identical bits to the device-resident call
    out_d, info_d, _ = run_gpu(n, batch, chunk, inter)
    assert np.array_equal(out.view(np.uint32), out_d.view(np.uint32))
    assert np.array_equal(info, info_d)


def test_host_end_to_end_pageable_memory():
    n, chunk, batch = 10, 32, 999
    canon, inter = make_batch(n, batch, chunk, kind="als")
    import torch
    hA = torch.from_numpy(inter.copy())          # not pinned
    hinfo = torch.zeros(batch, dtype=torch.int32)
    nf = bsp.batch_spotrf_interleaved_host(n, batch, chunk, hA, hinfo, slab=256)
    assert nf == 0
    assert_parity(n, batch, chunk, canon, inter, hA.numpy(), hinfo.numpy(), nf)
