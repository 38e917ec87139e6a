"""Pins of the FP64 oracle against what the definition and mathematics fix.

Each test names the pin and is chosen so that a
plausible mistake in oracle/cholesky.c -- a dropped update term, a wrong sign,
a swapped index or operand, a missing square root, a wrong pivot rule, an
off-by-one in info -- fails at least one of them.  No expected value here
comes from the CUDA path.
"""
import json
import math
import os

import numpy as np
import pytest

import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden", "handworked_p1.json")


def canon(M):
    """(n, n) or (B, n, n) math-indexed [i, j] -> canonical flat i + j*n."""
    M = np.asarray(M, dtype=np.float64)
    if M.ndim == 2:
        M = M[None]
    return np.ascontiguousarray(M.transpose(0, 2, 1)).reshape(M.shape[0], -1)


def mat(n, flat):
    """canonical flat -> [b, i, j]."""
    return np.asarray(flat).reshape(-1, n, n).transpose(0, 2, 1)


# ---------------------------------------------------------------- P1
def test_p1_handworked_exact(oracle_mod):
    d = json.load(open(GOLD))
    for c in d["cases"]:
        A = np.array(c["A"], dtype=np.float32)
        n = A.shape[0]
        L, info = oracle_mod.potrf(n, canon(A).astype(np.float32))
        assert info[0] == 0
        assert np.array_equal(mat(n, L)[0], np.array(c["L"], dtype=np.float64))


def test_p1_handworked_info(oracle_mod):
    d = json.load(open(GOLD))["info_cases"]
    for c in d["cases"]:
        A = np.array(c["A"], dtype=np.float32)
        n = A.shape[0]
        _, info = oracle_mod.potrf(n, canon(A).astype(np.float32))
        assert info[0] == c["info"], c


# ---------------------------------------------------------------- P2
@pytest.mark.parametrize("n", [1, 2, 3, 5, 8, 13, 16, 21, 24, 32, 33, 48, 64])
def test_p2_integer_factor_exact(oracle_mod, n):
    b = np.arange(64, dtype=np.uint64) + 1000
    A = synth.generate(n, "l0", 7, b, upper="nan")
    L0 = synth.l0_factor(n, 7, b)
    L, info = oracle_mod.potrf(n, A)
    assert (info == 0).all()
    assert np.array_equal(mat(n, L), L0)


@pytest.mark.parametrize("n", [1, 4, 16, 32, 64])
def test_p2_fig9_emulator_exact(oracle_mod, n):
    """The FP32 op-order emulator also returns exactly L0 (reading R3: the
    reciprocal-multiply of Fig. 9 is exact for power-of-two pivots)."""
    b = np.arange(64, dtype=np.uint64)
    A = synth.generate(n, "l0", 3, b, upper="nan")
    W, info = oracle_mod.spotrf_fig9_fp32(n, A)
    assert (info == 0).all()
    assert np.array_equal(mat(n, W).astype(np.float64), synth.l0_factor(n, 3, b))


# ---------------------------------------------------------------- P3
@pytest.mark.parametrize("n", [1, 2, 7, 32, 64])
def test_p3_identity_and_diagonal(oracle_mod, n):
    I = np.eye(n, dtype=np.float32)
    L, info = oracle_mod.potrf(n, canon(I).astype(np.float32))
    assert info[0] == 0 and np.array_equal(mat(n, L)[0], np.eye(n))
    d = (np.arange(n) % 9 + 1).astype(np.float64)
    D = np.diag(d * d).astype(np.float32)
    L, info = oracle_mod.potrf(n, canon(D).astype(np.float32))
    assert info[0] == 0 and np.array_equal(mat(n, L)[0], np.diag(d))


# ---------------------------------------------------------------- P4
@pytest.mark.parametrize("n", [2, 3, 10, 32, 64])
def test_p4_tridiag_toeplitz_minus1_2(oracle_mod, n):
    T = 2 * np.eye(n) - np.eye(n, k=1) - np.eye(n, k=-1)
    L, info = oracle_mod.potrf(n, canon(T).astype(np.float32))
    assert info[0] == 0
    L = mat(n, L)[0]
    k = np.arange(1, n + 1, dtype=np.float64)                  # 1-based
    assert np.allclose(np.diag(L), np.sqrt((k + 1) / k), rtol=0, atol=1e-14)
    kk = np.arange(1, n, dtype=np.float64)
    assert np.allclose(np.diag(L, -1), -np.sqrt(kk / (kk + 1)), rtol=0, atol=1e-14)
    assert np.count_nonzero(np.tril(L, -2)) == 0


@pytest.mark.parametrize("a,b", [(3.0, 1.0), (2.5, -1.0), (4.0, 1.5), (10.0, -0.5)])
@pytest.mark.parametrize("n", [5, 32, 64])
def test_p4_tridiag_general_sinh(oracle_mod, n, a, b):
    T = a * np.eye(n) + b * (np.eye(n, k=1) + np.eye(n, k=-1))
    L, info = oracle_mod.potrf(n, canon(T).astype(np.float32))
    assert info[0] == 0
    L = mat(n, L)[0]
    th = math.acosh(a / (2 * abs(b)))
    k = np.arange(1, n + 1, dtype=np.float64)
    d = abs(b) * np.sinh((k + 1) * th) / np.sinh(k * th)
    assert np.allclose(np.diag(L), np.sqrt(d), rtol=1e-13, atol=0)
    assert np.allclose(np.diag(L, -1), b / np.sqrt(d[:-1]), rtol=1e-13, atol=0)


# ---------------------------------------------------------------- P5
@pytest.mark.parametrize("n", [1, 2, 3, 8, 17, 32, 33, 64])
def test_p5_info_equals_k_dd(oracle_mod, n):
    ks = range(n) if n <= 17 else sorted({0, 1, n // 2, n - 1})
    base = synth.generate(n, "dd", 11, np.arange(1, dtype=np.uint64))[0]
    for kk in ks:
        A = base.copy()
        A[kk + kk * n] = -1.0
        L, info = oracle_mod.potrf(n, A[None])
        assert info[0] == kk + 1


@pytest.mark.parametrize("n", [2, 9, 32, 64])
def test_p5_info_and_final_columns_l0(oracle_mod, n):
    """Schur pivot exactly -1 at kk; columns j < kk equal L0's (reading R2)."""
    b = np.arange(200, dtype=np.uint64)
    A = synth.generate(n, "l0", 5, b, upper="nan", fail_seed=9, fail_period=3)
    failed, kk = synth.fail_plan(n, 9, 3, b)
    assert failed.any() and (~failed).any()
    L, info = oracle_mod.potrf(n, A)
    assert np.array_equal(info, np.where(failed, kk + 1, 0))
    L0 = synth.l0_factor(n, 5, b)
    Lm = mat(n, L)
    for t in np.nonzero(failed)[0]:
        c = kk[t]
        assert np.array_equal(Lm[t][:, :c], L0[t][:, :c])


@pytest.mark.parametrize("n", [1, 4, 20])
def test_p5_zero_and_nan_pivot(oracle_mod, n):
    base = synth.generate(n, "dd", 2, np.arange(1, dtype=np.uint64))[0]
    for kk in sorted({0, n // 2, n - 1}):
        for bad in (0.0, np.nan):
            A = base.copy()
            A[kk + kk * n] = bad   # kk = 0: pivot exactly 0 / NaN; kk > 0: pivot <= 0 or NaN
            _, info = oracle_mod.potrf(n, A[None])
            assert info[0] == kk + 1


# ---------------------------------------------------------------- P6
@pytest.mark.parametrize("n", [1, 3, 8, 16, 31, 32, 47, 64])
def test_p6_lapack_dpotrf(oracle_mod, n):
    from scipy.linalg import lapack
    rng = np.random.default_rng(n)
    for trial in range(8):
        X = rng.standard_normal((n, n))
        A = (X @ X.T + (n * 0.1 if trial % 2 == 0 else -0.5) * np.eye(n)).astype(np.float32)
        A = np.tril(A) + np.tril(A, -1).T
        c, info_ref = lapack.dpotrf(A.astype(np.float64), lower=1, clean=1)
        L, info = oracle_mod.potrf(n, canon(A).astype(np.float32))
        assert info[0] == info_ref
        if info_ref == 0:
            Lm = mat(n, L)[0]
            err = np.abs(Lm - c).max(axis=0) / np.abs(c).max(axis=0)
            assert err.max() <= 1e-12


# ---------------------------------------------------------------- P7 / S7 / S8
@pytest.mark.parametrize("kind", ["dd", "als"])
@pytest.mark.parametrize("n", [1, 2, 16, 32, 64])
def test_p7_invariants(oracle_mod, n, kind):
    b = np.arange(50, dtype=np.uint64)
    A = synth.generate(n, kind, 2017, b, upper="mirror")
    L, info = oracle_mod.potrf(n, A)
    assert (info == 0).all()
    Lm = mat(n, L)
    assert (np.diagonal(Lm, axis1=1, axis2=2) > 0).all()
    assert np.count_nonzero(np.triu(Lm, 1)) == 0
    Am = mat(n, A).astype(np.float64)
    R = Am - Lm @ Lm.transpose(0, 2, 1)
    assert np.abs(R).max() <= 1e-12 * np.abs(Am).max()
    if n == 1:
        assert np.array_equal(Lm[:, 0, 0], np.sqrt(Am[:, 0, 0]))


def test_s7_upper_triangle_ignored(oracle_mod):
    n = 12
    b = np.arange(30, dtype=np.uint64)
    Am = synth.generate(n, "dd", 1, b, upper="mirror")
    An = synth.generate(n, "dd", 1, b, upper="nan")
    L1, i1 = oracle_mod.potrf(n, Am)
    L2, i2 = oracle_mod.potrf(n, An)
    assert np.array_equal(L1, L2) and np.array_equal(i1, i2)


def test_s8_quick_return(oracle_mod):
    L, info = oracle_mod.potrf(0, np.zeros((5, 0), np.float32))
    assert L.shape == (5, 0) and (info == 0).all()
    L, info = oracle_mod.potrf(4, np.zeros((0, 16), np.float32))
    assert L.shape == (0, 16) and info.shape == (0,)


def test_threads_do_not_change_result(oracle_mod):
    n = 10
    A = synth.generate(n, "als", 4, np.arange(333, dtype=np.uint64))
    L1, i1 = oracle_mod.potrf(n, A, nthreads=1)
    L2, i2 = oracle_mod.potrf(n, A, nthreads=7)
    assert np.array_equal(L1, L2) and np.array_equal(i1, i2)
