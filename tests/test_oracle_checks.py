"""Pins of the acceptance metrics (oracle/checks.py) and models (oracle/metrics.py)."""
import numpy as np
import pytest

import synth
from oracle import checks, metrics


def test_metrics_formulas():
    # n^3/3 flops -- e.g. n = 3 -> 9, n = 32 -> 10922.67
    assert metrics.flops_per_matrix(3) == 9.0
    assert abs(metrics.flops_per_matrix(32) - 32768 / 3) < 1e-9
    # lower triangle n(n+1)/2 floats read + written + 4-B info
    for n in (1, 8, 16, 32, 64):
        assert metrics.factor_bytes_per_matrix(n) == 2 * 4 * (n * (n + 1) // 2) + 4
    assert metrics.factor_bytes_per_matrix(32) == 4228        # SURVEY table
    assert metrics.convert_bytes_per_matrix(16) == 2048


@pytest.mark.parametrize("n", [1, 5, 16, 32])
def test_checks_accept_exact_and_reject_mistakes(oracle_mod, n):
    b = np.arange(40, dtype=np.uint64)
    A = synth.generate(n, "dd", 1, b, upper="nan")
    L64, info = oracle_mod.potrf(n, A)
    L32 = L64.astype(np.float32)
    r = checks.accept(n, A, L32, info, L64, info)
    assert r["ok"].all()
    assert r["err"].max() <= 2 ** -24 * 1.01
    assert r["resid"].max() < 1.0
    if n == 1:
        return
    # a transposed factor (upper instead of lower) must fail O2 and O3
    M = L64.reshape(-1, n, n)
    T = np.ascontiguousarray(M.transpose(0, 2, 1)).reshape(-1, n * n)
    assert not checks.accept(n, A, T, info, L64, info)["ok"].any()
    # a sign flip in one subdiagonal entry fails
    bad = L32.copy()
    bad[:, 1] = -bad[:, 1]
    assert not checks.accept(n, A, bad, info, L64, info)["ok"].any()
    # wrong info fails O1
    assert not checks.accept(n, A, L32, info + 1, L64, info)["ok"].any()
    # NaN anywhere in a final column fails
    bad = L32.copy()
    bad[:, 0] = np.nan
    assert not checks.accept(n, A, bad, info, L64, info)["ok"].any()


def test_colnorm_ignores_columns_past_failure(oracle_mod):
    n = 8
    A = synth.generate(n, "dd", 1, np.arange(1, dtype=np.uint64), upper="mirror")
    A[0, 5 + 5 * n] = -1.0
    L64, info = oracle_mod.potrf(n, A)
    assert info[0] == 6
    L = L64.astype(np.float32)
    L[0, 5 + 5 * n:] = 123.0           # columns >= info-1 are unspecified (R2)
    assert checks.colnorm_error(n, L, L64, info)[0] <= 1e-6
    L[0, 4 * n + 4] += 1.0             # column 4 is final: must be caught
    assert checks.colnorm_error(n, L, L64, info)[0] > 1e-4


def test_upper_bits_unchanged():
    n = 4
    A = synth.generate(n, "dd", 1, np.arange(3, dtype=np.uint64), upper="nan")
    B = A.copy()
    B[:, 0] = 5.0                        # (0,0) is lower -> still unchanged upper
    assert checks.upper_bits_unchanged(n, A, B).all()
    B[1, 0 + 2 * n] = 1.0                # (0,2) is strict upper
    assert checks.upper_bits_unchanged(n, A, B).tolist() == [True, False, True]


# ---- hand-derived values of the normalised metrics (VERDICT r1 "unpinned") ----
# Each case perturbs an exact factor by one representable delta and derives the
# residual in closed form by hand, so a dropped n, eps = 2^-24 instead of 2^-23
# (reading R11), a missing symmetrisation or a wrong norm changes the number.

def _canon(M):
    M = np.asarray(M, dtype=np.float64)
    return np.ascontiguousarray(M.T).reshape(1, -1)


def test_residual_handworked_2x2():
    # A = [[4,2],[2,10]] (P1), L' = [[2,0],[1,3+d]], d = 2^-20 (3+d exact in FP32).
    # L'L'^T = [[4,2],[2,1+(3+d)^2]] -> R = diag(0, -(6d+d^2)), ||R||_F = 6d+d^2;
    # ||A||_F = sqrt(16+4+4+100) = sqrt(124); n = 2.
    d = 2.0 ** -20
    A = _canon([[4, 2], [np.nan, 10]]).astype(np.float32)   # canonical: (0,1) is the NaN upper
    A[0, 2] = np.nan
    A[0, 1] = 2
    Lp = _canon([[2, 7.0], [1, 3 + d]]).astype(np.float32)   # upper garbage must be ignored
    expected = (6 * d + d * d) / (2 * np.sqrt(124.0) * 2.0 ** -23)
    got = checks.residual(2, A, Lp)[0]
    assert abs(got - expected) <= 1e-12 * expected
    assert abs(expected - 2.1553) < 1e-3                    # 24 / (2 sqrt(124)) ~ 2.155


def test_residual_handworked_3x3():
    # A = [[4,12,-16],[12,37,-43],[-16,-43,98]], L = [[2,0,0],[6,1,0],[-8,5,3]] (P1).
    # L'[2,1] = 5+d, d = 2^-18: (L'L'^T)_21 = -48+(5+d) -> R_21 = R_12 = -d,
    # (L'L'^T)_22 = 64+(5+d)^2+9 -> R_22 = -(10d+d^2); other entries exact.
    # ||R||_F = sqrt(2 d^2 + (10d+d^2)^2); ||A||_F^2 = 416 + 3362 + 11709 = 15487; n = 3.
    d = 2.0 ** -18
    A = _canon([[4, 12, -16], [12, 37, -43], [-16, -43, 98]]).astype(np.float32)
    Lp = _canon([[2, 0, 0], [6, 1, 0], [-8, 5 + d, 3]]).astype(np.float32)
    expected = np.sqrt(2 * d * d + (10 * d + d * d) ** 2) / (3 * np.sqrt(15487.0) * 2.0 ** -23)
    got = checks.residual(3, A, Lp)[0]
    assert abs(got - expected) <= 1e-12 * expected
    assert 0.86 < expected < 0.87                       # sqrt(102) * 32 / (3 sqrt(15487))
    # the exact factor gives exactly zero
    L = _canon([[2, 0, 0], [6, 1, 0], [-8, 5, 3]]).astype(np.float32)
    assert checks.residual(3, A, L)[0] == 0.0


def test_solve_residual_handworked():
    # A (3x3 above), nrhs = 2, X = [x1 | x2], x1 = [1,-2,3], x2 = [2,1,-1]:
    # b1 = A x1 = [-68,-191,364], b2 = A x2 = [36,104,-173] (hand-multiplied).
    # Perturb x1_3 by d and x2_1 by d (d = 2^-20): r1 = -d A[:,2], ||r1||_inf = 98 d;
    # r2 = -d A[:,0], ||r2||_inf = 16 d.  ||A||_inf = max(32, 92, 157) = 157.
    # e_r = ||r||_inf / ((||A||_inf ||x_r||_inf + ||b_r||_inf) n eps), max over r.
    d = 2.0 ** -20
    A = _canon([[4, 12, -16], [12, 37, -43], [-16, -43, 98]]).astype(np.float32)
    Am = np.array([[4, 12, -16], [12, 37, -43], [-16, -43, 98]], np.float64)
    x1, x2 = np.array([1.0, -2, 3]), np.array([2.0, 1, -1])
    assert (Am @ x1).tolist() == [-68, -191, 364] and (Am @ x2).tolist() == [36, 104, -173]
    B = np.concatenate([[-68, -191, 364], [36, 104, -173]]).astype(np.float32)[None]
    X = np.concatenate([[1, -2, 3 + d], [2 + d, 1, -1]])[None]       # element (i, r) at i + 3r
    e1 = 98 * d / ((157 * (3 + d) + 364) * 3 * 2.0 ** -23)
    e2 = 16 * d / ((157 * (2 + d) + 173) * 3 * 2.0 ** -23)
    got = checks.solve_residual(3, 2, A, X, B)[0]
    assert abs(got - max(e1, e2)) <= 1e-12 * e1
    assert abs(e1 - 784 / 2505) < 1e-6                  # 98 * 8 / (835 * 3)
    # exact X -> 0; only the first column perturbed -> still e1 (max over columns)
    X0 = np.concatenate([[1, -2, 3], [2, 1, -1]]).astype(np.float64)[None]
    assert checks.solve_residual(3, 2, A, X0, B)[0] == 0.0
    X2 = X0.copy()
    X2[0, 3] += d
    assert abs(checks.solve_residual(3, 2, A, X2, B)[0] - e2) <= 1e-12 * e2


def test_strict_relative_error_handworked():
    # L64 columns (lower): c0 = [4, 0.02, -1], c1 = [2, 0.5], c2 = [1].
    # Column maxima 4, 2, 1 -> floor 1e-2 * max keeps |entry| >= 0.04, 0.02, 0.01:
    # entry (1,0) = 0.02 < 0.04 is excluded.
    L64 = _canon([[4, 0, 0], [0.02, 2, 0], [-1, 0.5, 1]])
    Lt = _canon([[4.004, 9, 9], [0.03, 2, 9], [-1.001, 0.5005, 1.002]])   # upper ignored
    # kept relative errors: (0,0) 1e-3, (2,0) 1e-3, (2,1) 1e-3, (2,2) 2e-3
    got = checks.strict_relative_error(3, Lt, L64, np.array([0]))[0]
    assert abs(got - 2e-3) < 1e-12
    # info = 3 -> only columns j < 2 are final: max 1e-3
    got = checks.strict_relative_error(3, Lt, L64, np.array([3]))[0]
    assert abs(got - 1e-3) < 1e-12
    # without the floor, (1,0) would give 0.5; the column-normalised O2 gives
    # max(0.01/4, 0.0005/2, 0.002/1) = 0.0025 -- both differ from the strict value
    assert abs(checks.colnorm_error(3, Lt, L64, np.array([0]))[0] - 0.0025) < 1e-12
