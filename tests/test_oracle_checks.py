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
