"""Pins of the FP64 solve oracle (oracle.potrs) -- SURVEY §8(f) f1."""
import json
import os

import numpy as np
import pytest

import synth
from oracle import checks

GOLD = os.path.join(os.path.dirname(__file__), "golden", "handworked_solve_p11.json")


def canon(M):
    M = np.asarray(M, dtype=np.float64)
    if M.ndim == 2:
        M = M[None]
    return np.ascontiguousarray(M.transpose(0, 2, 1)).reshape(M.shape[0], -1)


def test_p11_handworked(oracle_mod):
    for c in json.load(open(GOLD))["cases"]:
        A = np.array(c["A"], dtype=np.float64)
        X = np.array(c["X"], dtype=np.float64)
        B = np.array(c["B"], dtype=np.float64)
        assert np.array_equal(A @ X, B)
        n, nrhs = X.shape
        L, info = oracle_mod.potrf(n, canon(A).astype(np.float32))
        assert info[0] == 0
        Xo = oracle_mod.potrs(n, nrhs, L, canon(B).astype(np.float32))
        assert np.array_equal(Xo.reshape(nrhs, n).T, X)


@pytest.mark.parametrize("n", [1, 2, 5, 16, 32, 64])
@pytest.mark.parametrize("nrhs", [1, 3])
def test_integer_system_exact(oracle_mod, n, nrhs):
    """A = L0 L0^T, integer X in [-3, 3]: B = A X is an exact integer and the
    substitutions only divide by powers of two -> X recovered exactly."""
    bidx = np.arange(40, dtype=np.uint64)
    A = synth.generate(n, "l0", 3, bidx, upper="nan")
    L0 = synth.l0_factor(n, 3, bidx)
    rng = np.random.default_rng(n)
    X = rng.integers(-3, 4, size=(len(bidx), n, nrhs)).astype(np.float64)
    B = L0 @ (L0.transpose(0, 2, 1) @ X)
    assert np.abs(B).max() < 2 ** 24
    L, info = oracle_mod.potrf(n, A)
    Bc = np.ascontiguousarray(B.transpose(0, 2, 1)).reshape(len(bidx), -1).astype(np.float32)
    Xo = oracle_mod.potrs(n, nrhs, L, Bc).reshape(len(bidx), nrhs, n).transpose(0, 2, 1)
    assert np.array_equal(Xo, X)


@pytest.mark.parametrize("n", [1, 3, 8, 17, 32, 64])
def test_identity_and_diagonal(oracle_mod, n):
    I = np.eye(n)
    L, _ = oracle_mod.potrf(n, canon(I).astype(np.float32))
    b = np.arange(1, n + 1, dtype=np.float32)[None]
    assert np.array_equal(oracle_mod.potrs(n, 1, L, b)[0], b[0].astype(np.float64))
    d = (np.arange(n) % 5 + 1).astype(np.float64)
    L, _ = oracle_mod.potrf(n, canon(np.diag(d * d)).astype(np.float32))
    x = oracle_mod.potrs(n, 1, L, (d * d * 3).astype(np.float32)[None])[0]
    assert np.array_equal(x, np.full(n, 3.0))


@pytest.mark.parametrize("n", [2, 9, 24, 33, 64])
def test_lapack_dpotrs(oracle_mod, n):
    from scipy.linalg import lapack
    A = synth.generate(n, "als", 11, np.arange(20, dtype=np.uint64))
    L, info = oracle_mod.potrf(n, A)
    assert (info == 0).all()
    rng = np.random.default_rng(n)
    B = rng.standard_normal((20, n * 2)).astype(np.float32)
    X = oracle_mod.potrs(n, 2, L, B)
    for t in range(20):
        Lm = L[t].reshape(n, n).T
        ref, inf2 = lapack.dpotrs(Lm, B[t].reshape(2, n).T.astype(np.float64), lower=1)
        assert inf2 == 0
        assert np.abs(X[t].reshape(2, n).T - ref).max() <= 1e-12 * np.abs(ref).max()
    r = checks.solve_residual(n, 2, A, X, B)
    assert r.max() < 1e-6          # FP64 solve: far below the FP32 bound of 10


def test_solve_checks_catch_mistakes(oracle_mod):
    n = 6
    A = synth.generate(n, "dd", 1, np.arange(10, dtype=np.uint64))
    L, _ = oracle_mod.potrf(n, A)
    B = np.random.default_rng(0).standard_normal((10, n)).astype(np.float32)
    X = oracle_mod.potrs(n, 1, L, B)
    assert checks.solve_residual(n, 1, A, X.astype(np.float32), B).max() < 10
    assert (checks.solve_residual(n, 1, A, -X, B) > 10).all()
    Xw = X.copy()
    Xw[:, 0] += 1e-3 * np.abs(X).max()
    assert (checks.solve_residual(n, 1, A, Xw, B) > 10).all()
    assert checks.solve_forward_error(n, 1, X, X).max() == 0
