"""GPU parity: the CUDA path (through the C ABI) against the FP64 oracle.

Bar: info bit-exact (O1); column-normalised factor error
<= 1e-4 (O2, reading R10); scaled residual <= 10 (O3, R11); strict upper
triangle and pad lanes bitwise untouched (O4); and -- stronger than the bar --
bitwise equality with the FP32 Fig. 9 op-order emulator (P8).
"""
import numpy as np
import pytest

import oracle
import synth
from oracle import layout

import paper_conf_ipps_gatesklpd17_b200 as bsp
from gpu_helpers import assert_parity, make_batch, run_gpu, torch_mod

pytestmark = pytest.mark.gpu

ALL_N = list(range(1, 33)) + [33, 37, 40, 48, 56, 63, 64]


@pytest.mark.parametrize("n", ALL_N)
def test_parity_chunk32_ragged(n):
    batch = 3 * 128 + 37          # several blocks / chunks and a ragged tail
    canon, inter = make_batch(n, batch, 32, kind="dd")
    out, info, cnt = run_gpu(n, batch, 32, inter)
    assert_parity(n, batch, 32, canon, inter, out, info, cnt)


@pytest.mark.parametrize("n", [1, 2, 5, 8, 13, 16, 20, 21, 24, 27, 32, 40, 64])
@pytest.mark.parametrize("chunk", [0, 64, 128, 256, 96])
def test_parity_other_chunks(n, chunk):
    batch = 301
    canon, inter = make_batch(n, batch, chunk, kind="als", seed=5)
    out, info, cnt = run_gpu(n, batch, chunk, inter)
    assert_parity(n, batch, chunk, canon, inter, out, info, cnt)


@pytest.mark.parametrize("n", [1, 3, 8, 16, 21, 25, 32, 33, 64])
def test_info_exact_with_injected_failures(n):
    batch = 777
    canon, inter = make_batch(n, batch, 32, kind="dd", fail_seed=2018, fail_period=7)
    failed, kk = synth.fail_plan(n, 2018, 7, np.arange(batch, dtype=np.uint64))
    out, info, cnt = run_gpu(n, batch, 32, inter)
    assert np.array_equal(info, np.where(failed, kk + 1, 0))
    assert cnt == int(failed.sum())
    assert_parity(n, batch, 32, canon, inter, out, info, cnt)


@pytest.mark.parametrize("n", [1, 4, 9, 16, 24, 32, 48, 64])
def test_integer_factor_bit_exact(n):
    """P2: A = L0 L0^T with integer L0 -> the GPU returns exactly L0."""
    batch = 200
    canon, inter = make_batch(n, batch, 32, kind="l0", seed=9)
    out, info, _ = run_gpu(n, batch, 32, inter)
    assert (info == 0).all()
    got = layout.from_interleaved(n, batch, 32, out).reshape(-1, n, n).transpose(0, 2, 1)
    L0 = synth.l0_factor(n, 9, np.arange(batch, dtype=np.uint64))
    assert np.array_equal(np.tril(got).astype(np.float64), L0)


def _panel_s(n):
    return [s for s in range(4, n - 7, 4) if n - s <= 16] if 20 <= n <= 32 else []


def _ptmem_s(n):
    import sys, os
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "scripts"))
    import gen_instances
    return gen_instances.ptmem_s_values(n)


def gen_instances_mod():
    import sys, os
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "scripts"))
    import gen_instances
    return gen_instances


def _qtm_combos(n):
    import sys, os
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "scripts"))
    import gen_instances
    if n not in gen_instances.QTM_N:
        return []
    return [(p_, c, pre) for p_, c, pre in gen_instances.QTM_COMBOS if gen_instances.qtm_fits(n, p_, c, pre)]


@pytest.mark.parametrize("n", [33, 35, 38, 44, 45, 47, 50, 53, 57, 60, 62, 64])
@pytest.mark.parametrize("chunk", [32, 0, 96])
def test_qtm_parity_failures_ragged(n, chunk):
    """Variant QTM (P threads per matrix, matrix on chip): every (P, TMEM
    columns) instance against the oracle, with injected failures, a batch that
    is not a multiple of the matrices per CTA, and the runtime-stride path."""
    batch = 3 * 32 + 13
    canon, inter = make_batch(n, batch, chunk, kind="dd", seed=n, fail_seed=2018, fail_period=5)
    failed, kk = synth.fail_plan(n, 2018, 5, np.arange(batch, dtype=np.uint64))
    combos = _qtm_combos(n)
    ts = [dict(variant=bsp.VARIANT_QTM, threads_per_block=128, param=p_,
               staging=gen_instances_mod().qtm_staging(cols, pre)) for p_, cols, pre in combos]
    ts = [t for t in ts if bsp.bspotrf_tuning_available(n, chunk, t)]
    assert ts                                      # the core build keeps one QTM point per n
    for t in ts:
        out, info, cnt = run_gpu(n, batch, chunk, inter, tune=t)
        assert np.array_equal(info, np.where(failed, kk + 1, 0)), t
        assert_parity(n, batch, chunk, canon, inter, out, info, cnt)


def _rcw_ncta(n):
    g = gen_instances_mod()
    return g.rcw_ncta(n) if n in g.RCW_N else ()


@pytest.mark.parametrize("n", [33, 34, 39, 40, 41, 47, 48, 49, 55, 56, 57, 61, 63, 64])
@pytest.mark.parametrize("chunk", [32, 0, 96])
def test_rcw_parity_failures_ragged(n, chunk):
    """Variant RCW (8 warps share 32 matrices, factor in TMEM): every CTAs-per-SM
    instance against the oracle and bitwise against the Fig. 9 emulator, with
    injected failures, a batch that is not a multiple of 32, every n mod 8, and
    the runtime-stride path (chunk 0, 96)."""
    batch = 5 * 32 + 13
    canon, inter = make_batch(n, batch, chunk, kind="dd", seed=n + 11, fail_seed=2018, fail_period=5)
    failed, kk = synth.fail_plan(n, 2018, 5, np.arange(batch, dtype=np.uint64))
    assert _rcw_ncta(n)
    ts = [dict(variant=bsp.VARIANT_RCW, threads_per_block=256, param=k, staging=0) for k in _rcw_ncta(n)]
    if n in gen_instances_mod().RCW16_N:
        ts.append(dict(variant=bsp.VARIANT_RCW16, threads_per_block=512, param=0, staging=0))
    if n in gen_instances_mod().RCWD_N:
        ts.append(dict(variant=bsp.VARIANT_RCWD, threads_per_block=288, param=0, staging=0))
    if n in gen_instances_mod().RCWP_N:
        ts += [dict(variant=bsp.VARIANT_RCWP, threads_per_block=256, param=d1, staging=0)
               for d1 in gen_instances_mod().rcwp_params(n)]
    for t in ts:
        out, info, cnt = run_gpu(n, batch, chunk, inter, tune=t)
        assert np.array_equal(info, np.where(failed, kk + 1, 0)), t
        assert_parity(n, batch, chunk, canon, inter, out, info, cnt)


@pytest.mark.parametrize("n", [33, 49, 57, 64])
@pytest.mark.parametrize("chunk,batch", [(0, 5 * 32 + 12), (0, 4 * 2 * 148 * 32 + 44), (64, 5 * 32 + 12),
                                         (160, 3 * 160 + 37)])
def test_rcwp_tma2d_runtime_chunk(n, chunk, batch):
    """RCWP at runtime chunks whose stride is a multiple of 16 B stages each
    column block by 2-D TMA boxes (32 matrices x (N - 8c) rows) from one tensor
    map per block: against the oracle and bitwise against RCW, with failures, a
    partial last group (chunk 0: the box runs past the row end and is
    zero-filled; other chunks: pad lanes) and, at the large batch, several
    groups per persistent CTA."""
    canon, inter = make_batch(n, batch, chunk, kind="dd", seed=n + 3, fail_seed=2018, fail_period=7)
    failed, kk = synth.fail_plan(n, 2018, 7, np.arange(batch, dtype=np.uint64))
    ref = None
    for t in [dict(variant=bsp.VARIANT_RCWP, threads_per_block=256, param=d1, staging=0)
               for d1 in gen_instances_mod().rcwp_params(n)] + \
             [dict(variant=bsp.VARIANT_RCW, threads_per_block=256, param=_rcw_ncta(n)[0], staging=0)]:
        out, info, cnt = run_gpu(n, batch, chunk, inter, tune=t)
        assert np.array_equal(info, np.where(failed, kk + 1, 0)), t
        if ref is None:
            if batch < 10000:
                assert_parity(n, batch, chunk, canon, inter, out, info, cnt)
            ref = out
        else:
            assert np.array_equal(out.view(np.uint32), ref.view(np.uint32)), t


@pytest.mark.parametrize("n", [36, 48, 52, 64])
def test_rcw_integer_and_als(n):
    """RCW on the exactness set (P2: returns exactly L0) and on ALS-shaped input."""
    batch = 2 * 32 + 5
    for k in _rcw_ncta(n):
        t = dict(variant=bsp.VARIANT_RCW, threads_per_block=256, param=k, staging=0)
        canon, inter = make_batch(n, batch, 32, kind="l0", seed=9)
        out, info, _ = run_gpu(n, batch, 32, inter, tune=t)
        assert (info == 0).all()
        got = layout.from_interleaved(n, batch, 32, out).reshape(-1, n, n).transpose(0, 2, 1)
        L0 = synth.l0_factor(n, 9, np.arange(batch, dtype=np.uint64))
        assert np.array_equal(np.tril(got).astype(np.float64), L0)
        canon, inter = make_batch(n, batch, 32, kind="als", seed=4)
        out, info, cnt = run_gpu(n, batch, 32, inter, tune=t)
        assert_parity(n, batch, 32, canon, inter, out, info, cnt)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 6, 7, 8])
@pytest.mark.parametrize("chunk,batch", [(32, 3 * 512 + 37), (0, 4 * 301), (0, 4 * 301 + 1), (96, 999), (64, 2)])
def test_regv_128bit_groups(n, chunk, batch):
    """Variant REGV (4 adjacent matrices per thread, float4 accesses): bitwise equal to
    the Fig. 9 emulator and O1-O4 (pad lanes untouched when a group straddles the end
    of the batch), with injected failures; chunk 0 with batch % 4 != 0 takes the REG
    fallback."""
    canon, inter = make_batch(n, batch, chunk, kind="dd", seed=n + 21, fail_seed=2018, fail_period=6)
    failed, kk = synth.fail_plan(n, 2018, 6, np.arange(batch, dtype=np.uint64))
    for tpb in (64, 128):
        t = dict(variant=bsp.VARIANT_REGV, threads_per_block=tpb, param=0, staging=0)
        out, info, cnt = run_gpu(n, batch, chunk, inter, tune=t)
        assert np.array_equal(info, np.where(failed, kk + 1, 0)), t
        assert_parity(n, batch, chunk, canon, inter, out, info, cnt)


@pytest.mark.parametrize("n", [1, 2, 3, 5, 8, 11, 12, 16])
@pytest.mark.parametrize("chunk", [32, 0, 96])
def test_regx_multi_matrix_and_fast_math(n, chunk):
    """Variant REGX: M matrices per thread (IEEE: bitwise equal to
    the Fig. 9 emulator) and the fast-math form (reading R4: O1-O4 only, exempt from
    the bitwise pins), with injected failures and a ragged batch."""
    batch = 2 * 128 * 4 + 77
    canon, inter = make_batch(n, batch, chunk, kind="als", seed=n + 3, fail_seed=2018, fail_period=9)
    failed, kk = synth.fail_plan(n, 2018, 9, np.arange(batch, dtype=np.uint64))
    for m, fast in gen_instances_mod().regx_combos(n):
        for tpb in (64, 128):
            t = dict(variant=bsp.VARIANT_REGX, threads_per_block=tpb, param=m, staging=int(fast))
            out, info, cnt = run_gpu(n, batch, chunk, inter, tune=t)
            assert np.array_equal(info, np.where(failed, kk + 1, 0)), t
            assert_parity(n, batch, chunk, canon, inter, out, info, cnt, emulate=not fast)


def _tunings(n, chunk):
    out = []
    if n <= 24:
        for tpb in (32, 64, 128, 256):
            out.append(dict(variant=bsp.VARIANT_REG, threads_per_block=tpb, param=0, staging=0))
    if 11 <= n <= 17:
        out.append(dict(variant=bsp.VARIANT_REG, threads_per_block=128, param=12, staging=0))
    for s in _panel_s(n):
        out.append(dict(variant=bsp.VARIANT_PANEL, threads_per_block=32, param=s, staging=2))
        out.append(dict(variant=bsp.VARIANT_PANEL, threads_per_block=64, param=s, staging=2))
        if chunk in (32, 64, 128):
            out.append(dict(variant=bsp.VARIANT_PANEL, threads_per_block=0, param=s, staging=1))
    if 4 <= n <= 20 and chunk == 32:
        for w in (2, 4):
            out.append(dict(variant=bsp.VARIANT_RTMA, threads_per_block=0, param=w, staging=1))
            out.append(dict(variant=bsp.VARIANT_RTMAP, threads_per_block=0, param=w, staging=1))
    if 24 <= n <= 44:
        for s in _ptmem_s(n):
            out.append(dict(variant=bsp.VARIANT_PTMEM, threads_per_block=128, param=s, staging=2))
            if chunk == 32:
                out.append(dict(variant=bsp.VARIANT_PTMEM, threads_per_block=128, param=s, staging=1))
                out.append(dict(variant=bsp.VARIANT_PTMEM, threads_per_block=128, param=s, staging=3))
    for m, fast in gen_instances_mod().regx_combos(n) if n in gen_instances_mod().REGX_N else []:
        if not fast:                              # IEEE: same op sequence -> same bits
            out.append(dict(variant=bsp.VARIANT_REGX, threads_per_block=128, param=m, staging=0))
    for p_, cols, pre in _qtm_combos(n):
        out.append(dict(variant=bsp.VARIANT_QTM, threads_per_block=128, param=p_,
                        staging=gen_instances_mod().qtm_staging(cols, pre)))
    for k in _rcw_ncta(n):
        out.append(dict(variant=bsp.VARIANT_RCW, threads_per_block=256, param=k, staging=0))
    if n in gen_instances_mod().RCW16_N:
        out.append(dict(variant=bsp.VARIANT_RCW16, threads_per_block=512, param=0, staging=0))
    if n in gen_instances_mod().RCWD_N:
        out.append(dict(variant=bsp.VARIANT_RCWD, threads_per_block=288, param=0, staging=0))
    if n in gen_instances_mod().RCWP_N:
        out += [dict(variant=bsp.VARIANT_RCWP, threads_per_block=256, param=d1, staging=0)
               for d1 in gen_instances_mod().rcwp_params(n)]
    if n <= 8:
        out.append(dict(variant=bsp.VARIANT_REGV, threads_per_block=128, param=0, staging=0))
    for tpb in (64, 256):
        for nb in (2, 4, 8):
            if nb <= n or nb == 2:
                out.append(dict(variant=bsp.VARIANT_TILE, threads_per_block=tpb, param=nb, staging=0))
    if 17 <= n <= 32:
        for s in (n - 16, n - 14, n - 12):
            if 2 <= s <= n - 2:
                out.append(dict(variant=bsp.VARIANT_SMEM, threads_per_block=32, param=s, staging=2))
                out.append(dict(variant=bsp.VARIANT_SMEM, threads_per_block=64, param=s, staging=2))
                if chunk in (32, 64, 128):
                    out.append(dict(variant=bsp.VARIANT_SMEM, threads_per_block=0, param=s, staging=1))
    # the default (core) build holds a subset of the sweep space: test every
    # instance it has (BSPOTRF_SWEEP=1 builds all of them)
    return [t for t in out if bsp.bspotrf_tuning_available(n, chunk, t)]


@pytest.mark.parametrize("n", [2, 7, 13, 16, 19, 20, 21, 23, 24, 25, 27, 28, 29, 30, 31, 32, 33, 36, 39,
                               40, 44, 45, 49, 56, 61, 64])
@pytest.mark.parametrize("chunk", [32, 64, 0])
def test_all_variants_bitwise_identical(n, chunk):
    """P8: every variant / staging / block size gives the same bits."""
    batch = 2 * 128 + 19
    canon, inter = make_batch(n, batch, chunk, kind="als", seed=77)
    ref = None
    ts = _tunings(n, chunk)
    table = bsp.bspotrf_get_tuning(n, chunk).as_dict()
    variants = {t["variant"] for t in ts}
    assert len(ts) >= 3 and len(variants) >= 2, ts
    ts.append(table)                               # the table's own choice, whatever it is
    for t in ts:
        out, info, cnt = run_gpu(n, batch, chunk, inter, tune=t)
        if ref is None:
            assert_parity(n, batch, chunk, canon, inter, out, info, cnt)
            ref = (out, info)
        else:
            assert np.array_equal(out.view(np.uint32), ref[0].view(np.uint32)), t
            assert np.array_equal(info, ref[1]), t


def test_quick_returns_touch_nothing():
    torch = torch_mod()
    A = torch.full((64,), 3.0, device="cuda")
    info = torch.full((4,), 5, dtype=torch.int32, device="cuda")
    bsp.batch_spotrf_interleaved(0, 4, 32, A, info)
    bsp.batch_spotrf_interleaved(4, 0, 32, A, info)
    torch.cuda.synchronize()
    assert (A == 3.0).all() and (info == 5).all()


def test_single_matrix_and_tiny_batches():
    for batch in (1, 2, 31, 33):
        for n in (1, 2, 17, 32):
            canon, inter = make_batch(n, batch, 32, kind="dd", seed=batch)
            out, info, cnt = run_gpu(n, batch, 32, inter)
            assert_parity(n, batch, 32, canon, inter, out, info, cnt)


def test_nan_pivot_reported():
    n, batch = 6, 64
    canon, _ = make_batch(n, batch, 32, kind="dd", upper="mirror")
    canon[5, 3 + 3 * n] = np.nan
    canon[9, 0] = 0.0
    inter = layout.to_interleaved(n, 32, canon, fill_bits=synth.PAD_BITS)
    out, info, cnt = run_gpu(n, batch, 32, inter)
    assert info[5] == 4 and info[9] == 1 and cnt == 2
    assert (np.delete(info, [5, 9]) == 0).all()


@pytest.mark.parametrize("n", [40, 57, 64])
@pytest.mark.parametrize("chunk", [32, 0, 96])
def test_rcw_many_groups_per_cta(n, chunk):
    """RCW / RCW16 are persistent (one or two CTAs per SM): with more than
    2 * SMs * 32 matrices every CTA loops over several 32-matrix groups, so the
    next-group prefetch, the half flip and the mbarrier parity across groups
    are exercised, with a ragged tail.  Sampled matrices against the oracle
    (first/last groups of every CTA's walk are in the sample), the fused count
    exact, and RCW == RCW16 bitwise (P8)."""
    torch = torch_mod()
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    batch = 2 * sms * 32 * 3 + 77
    b = np.arange(batch, dtype=np.uint64)
    canon = synth.generate(n, "dd", 31, b, upper="nan", fail_seed=2018, fail_period=97)
    failed, kk = synth.fail_plan(n, 2018, 97, b)
    inter = layout.to_interleaved(n, chunk, canon, fill_bits=synth.PAD_BITS)
    ts = [dict(variant=bsp.VARIANT_RCW, threads_per_block=256, param=k, staging=0) for k in _rcw_ncta(n)]
    if n in gen_instances_mod().RCW16_N:
        ts.append(dict(variant=bsp.VARIANT_RCW16, threads_per_block=512, param=0, staging=0))
    if n in gen_instances_mod().RCWD_N:
        ts.append(dict(variant=bsp.VARIANT_RCWD, threads_per_block=288, param=0, staging=0))
    if n in gen_instances_mod().RCWP_N:
        ts += [dict(variant=bsp.VARIANT_RCWP, threads_per_block=256, param=d1, staging=0)
               for d1 in gen_instances_mod().rcwp_params(n)]
    idx = np.unique(np.concatenate([np.arange(0, batch, 37), np.arange(batch - 200, batch),
                                    np.arange(0, 64 * 32, 31)]))
    ref = None
    for t in ts:
        out, info, cnt = run_gpu(n, batch, chunk, inter, tune=t)
        assert np.array_equal(info, np.where(failed, kk + 1, 0)), t
        assert cnt == int(failed.sum())
        pads = layout.pad_lane_offsets(n, batch, chunk)
        assert np.array_equal(out.view(np.uint32)[pads], inter.view(np.uint32)[pads])
        got = layout.from_interleaved(n, batch, chunk, out)[idx]
        L64, info64 = oracle.potrf(n, canon[idx])
        from oracle import checks
        r = checks.accept(n, canon[idx], got, info[idx], L64, info64)
        assert r["ok"].all(), (t, np.nonzero(~r["ok"])[0][:5])
        if ref is None:
            ref = out
        else:
            assert np.array_equal(out.view(np.uint32), ref.view(np.uint32)), t


@pytest.mark.parametrize("n,chunk,variant,param", [(32, 64, 5, 16), (36, 0, 5, 20), (38, 160, 5, 24),
                                                   (40, 0, 14, 2), (48, 64, 14, 0), (51, 96, 14, 1)])
def test_tma2d_staging_bitwise_equal_to_cp_async(monkeypatch, n, chunk, variant, param):
    """Runtime-chunk staging by 2-D tensor TMA (PTMEM n = 32..38, RCWP n <= 51)
    and the per-thread cp.async form (BSPOTRF_TMA2D=0) give the same bits, and
    both pass the oracle, with failures and a partial last group."""
    batch = 7 * 32 + 20 if chunk == 0 else 7 * 32 + 19
    canon, inter = make_batch(n, batch, chunk, kind="als", seed=n, fail_seed=2018, fail_period=9)
    tune = dict(variant=variant, threads_per_block=128 if variant == 5 else 256, param=param,
                staging=2 if variant == 5 else 0)
    out1, info1, cnt1 = run_gpu(n, batch, chunk, inter, tune=tune)
    monkeypatch.setenv("BSPOTRF_TMA2D", "0")
    out0, info0, cnt0 = run_gpu(n, batch, chunk, inter, tune=tune)
    assert np.array_equal(out1.view(np.uint32), out0.view(np.uint32))
    assert np.array_equal(info1, info0) and cnt1 == cnt0
    assert_parity(n, batch, chunk, canon, inter, out1, info1, cnt1)
