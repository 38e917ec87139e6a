"""GPU: batched SPOTRS and fused SPOSV through the C ABI,
against the FP64 oracle solve."""
import numpy as np
import pytest

import oracle
import synth
from oracle import checks, layout

import paper_conf_ipps_gatesklpd17_b200 as bsp
from gpu_helpers import torch_mod

pytestmark = pytest.mark.gpu


def run_sposv(n, nrhs, batch, chunk, A_c, B_c, fused_api=True):
    torch = torch_mod()
    Ai = layout.to_interleaved(n, chunk, A_c, fill_bits=synth.PAD_BITS)
    Bi = layout.rect_to_interleaved(n, nrhs, chunk, B_c, fill_bits=synth.PAD_BITS)
    dA = torch.from_numpy(Ai.copy()).cuda()
    dB = torch.from_numpy(Bi.copy()).cuda()
    info = torch.full((batch,), -3, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    if fused_api:
        bsp.batch_sposv_interleaved(n, nrhs, batch, chunk, dA, dB, info, nfailed=cnt)
    else:
        bsp.batch_spotrf_interleaved_ex(n, batch, chunk, dA, info, nfailed=cnt)
        bsp.batch_spotrs_interleaved(n, nrhs, batch, chunk, dA, dB)
    torch.cuda.synchronize()
    return Ai, Bi, dA.cpu().numpy(), dB.cpu().numpy(), info.cpu().numpy(), int(cnt.item())


def check_solution(n, nrhs, batch, chunk, A_c, B_c, Ai, Bi, Aout, Bout, info):
    L64, info64 = oracle.potrf(n, A_c)
    assert np.array_equal(info, info64)
    L = layout.from_interleaved(n, batch, chunk, Aout)
    assert checks.accept(n, A_c, L, info, L64, info64)["ok"].all()
    X = layout.rect_from_interleaved(n, nrhs, batch, chunk, Bout)
    ok = info64 == 0
    X64 = oracle.potrs(n, nrhs, L64, B_c)
    r = checks.solve_residual(n, nrhs, A_c, X, B_c)
    assert r[ok].max(initial=0) <= 10.0, r.max()
    fe = checks.solve_forward_error(n, nrhs, X, X64)
    assert fe[ok].max(initial=0) <= 1e-4, fe.max()     # DD / ALS inputs: cond <= ~200
    # failed matrices keep their right-hand sides (LAPACK SPOSV semantics)
    if (~ok).any():
        assert np.array_equal(X[~ok].view(np.uint32), B_c[~ok].view(np.uint32))
    pads = np.setdiff1d(np.arange(Bi.size), layout.rect_offset(
        n, nrhs, batch, chunk, np.arange(batch)[:, None], (np.arange(n * nrhs) % n)[None, :],
        (np.arange(n * nrhs) // n)[None, :]).ravel())
    assert np.array_equal(Bout.view(np.uint32)[pads], Bi.view(np.uint32)[pads])
    return X


@pytest.mark.parametrize("n", [1, 2, 5, 8, 13, 16, 20, 21, 24, 29, 32, 33, 40, 44, 48, 64])
@pytest.mark.parametrize("nrhs", [1, 3, 5])
@pytest.mark.parametrize("chunk", [32, 0])
def test_sposv_matches_oracle(n, nrhs, chunk):
    batch = 2 * 128 + 21
    b = np.arange(batch, dtype=np.uint64)
    A_c = synth.generate(n, "als", 4, b, upper="nan", fail_seed=9, fail_period=13)
    B_c = synth.generate_rhs(n, nrhs, 5, b)
    Ai, Bi, Aout, Bout, info, cnt = run_sposv(n, nrhs, batch, chunk, A_c, B_c)
    check_solution(n, nrhs, batch, chunk, A_c, B_c, Ai, Bi, Aout, Bout, info)
    assert cnt == int((info != 0).sum()) > 0


@pytest.mark.parametrize("n,nrhs", [(3, 1), (3, 4), (8, 2), (16, 1), (16, 4), (20, 3),
                                    (24, 1), (25, 1), (28, 1), (31, 1), (32, 1), (33, 1), (36, 1),
                                    (40, 1), (44, 1)])
def test_fused_equals_factor_then_solve_bitwise(n, nrhs):
    batch = 300
    b = np.arange(batch, dtype=np.uint64)
    A_c = synth.generate(n, "dd", 8, b, upper="mirror")
    B_c = synth.generate_rhs(n, nrhs, 1, b)
    _, _, A1, B1, i1, _ = run_sposv(n, nrhs, batch, 32, A_c, B_c, fused_api=True)
    _, _, A2, B2, i2, _ = run_sposv(n, nrhs, batch, 32, A_c, B_c, fused_api=False)
    assert np.array_equal(A1.view(np.uint32), A2.view(np.uint32))
    assert np.array_equal(B1.view(np.uint32), B2.view(np.uint32))
    assert np.array_equal(i1, i2)


@pytest.mark.parametrize("n", [1, 4, 16, 20, 32, 64])
def test_integer_system_exact(n):
    """A = L0 L0^T and integer X: B = A X exact; the GPU returns X exactly."""
    batch, nrhs = 100, 2
    b = np.arange(batch, dtype=np.uint64)
    A_c = synth.generate(n, "l0", 6, b, upper="nan")
    L0 = synth.l0_factor(n, 6, b)
    rng = np.random.default_rng(n)
    X = rng.integers(-3, 4, size=(batch, n, nrhs)).astype(np.float64)
    Bm = L0 @ (L0.transpose(0, 2, 1) @ X)
    B_c = np.ascontiguousarray(Bm.transpose(0, 2, 1)).reshape(batch, -1).astype(np.float32)
    _, _, _, Bout, info, _ = run_sposv(n, nrhs, batch, 32, A_c, B_c)
    assert (info == 0).all()
    Xg = layout.rect_from_interleaved(n, nrhs, batch, 32, Bout).reshape(batch, nrhs, n).transpose(0, 2, 1)
    assert np.array_equal(Xg.astype(np.float64), X)


def test_solve_argument_errors():
    L = bsp.lib()
    fake = 0x1000
    assert L.batch_spotrs_interleaved(65, 1, 10, 32, fake, fake, None) == -1
    assert L.batch_spotrs_interleaved(4, -1, 10, 32, fake, fake, None) == -2
    assert L.batch_spotrs_interleaved(4, 1, -1, 32, fake, fake, None) == -3
    assert L.batch_spotrs_interleaved(4, 1, 10, 7, fake, fake, None) == -4
    assert L.batch_spotrs_interleaved(4, 1, 10, 32, None, fake, None) == -5
    assert L.batch_spotrs_interleaved(4, 1, 10, 32, fake, None, None) == -6
    assert L.batch_spotrs_interleaved(4, 0, 10, 32, None, None, None) == 0
    assert L.batch_sposv_interleaved(4, 1, 10, 32, fake, fake, None, None, None) == -7
