"""Acceptance metrics O1-O4, FP64, numpy.

TEST INFRASTRUCTURE (see oracle/__init__.py).

north_star: info bit-exact; factor within 1e-4 "max elementwise relative error"
against the FP64 oracle factor -- reading R10: normalised per
column, e_b = max_j max_{i>=j} |L_ij - L64_ij| / max_{i>=j} |L64_ij| -- and the
scaled backward residual ||A - L L^T||_F / (n ||A||_F eps_fp32) <= 10 with
eps_fp32 = 2^-23 (reading R11).  Arrays are canonical (batch, n*n), element
(i, j) at i + j*n.
"""
from __future__ import annotations

import numpy as np

EPS32 = 2.0 ** -23
FACTOR_TOL = 1e-4
RESID_TOL = 10.0
STRICT_TOL = 1e-4        # R10 diagnostic bar: the north star's literal 1e-4 on kept entries
STRICT_FLOOR = 1e-2      # entries >= STRICT_FLOOR * column max are kept


def _mats(n, X, dtype=np.float64):
    X = np.asarray(X).reshape(-1, n * n).astype(dtype)
    return X.reshape(-1, n, n).transpose(0, 2, 1)          # [b, i, j]


def lower_mask(n):
    return np.tril(np.ones((n, n), dtype=bool))


def colnorm_error(n, L_test, L64, info):
    """O2 per matrix.  Columns j < info-1 only when info > 0 (reading R2)."""
    Lt = _mats(n, L_test)
    Lr = _mats(n, L64)
    info = np.asarray(info).reshape(-1)
    low = lower_mask(n)[None]
    diff = np.where(low, np.abs(Lt - Lr), 0.0)
    diff = np.where(np.isnan(diff), np.inf, diff)
    ref = np.where(low, np.abs(Lr), 0.0)
    colmax = ref.max(axis=1)                                # [b, j]
    colerr = diff.max(axis=1)                               # [b, j]
    with np.errstate(divide="ignore", invalid="ignore"):
        rel = np.where(colmax > 0, colerr / colmax, np.where(colerr > 0, np.inf, 0.0))
    j = np.arange(n)[None, :]
    ncols = np.where(info > 0, np.maximum(info - 1, 0), n)[:, None]
    rel = np.where(j < ncols, rel, 0.0)
    return rel.max(axis=1) if n else np.zeros(len(info))


def strict_relative_error(n, L_test, L64, info, floor=STRICT_FLOOR):
    """Diagnostic: elementwise relative error restricted to |L64_ij| >=
    floor * column max (R10's literal reading is ill-posed for entries that
    come from cancellation)."""
    Lt = _mats(n, L_test)
    Lr = _mats(n, L64)
    info = np.asarray(info).reshape(-1)
    low = lower_mask(n)[None]
    colmax = np.where(low, np.abs(Lr), 0.0).max(axis=1, keepdims=True)
    keep = low & (np.abs(Lr) >= floor * colmax)
    j = np.arange(n)[None, None, :]
    ncols = np.where(info > 0, np.maximum(info - 1, 0), n)[:, None, None]
    keep = keep & (j < ncols)
    with np.errstate(divide="ignore", invalid="ignore"):
        rel = np.where(keep, np.abs(Lt - Lr) / np.abs(Lr), 0.0)
    return rel.reshape(len(info), -1).max(axis=1) if n else np.zeros(len(info))


def residual(n, A_in, L_test):
    """O3: ||sym(A) - L L^T||_F / (n ||sym(A)||_F eps32), FP64, from the FP32
    input's lower triangle (symmetrised) and the FP32 factor's lower triangle."""
    A = _mats(n, A_in)
    low = lower_mask(n)[None]
    Al = np.where(low, A, 0.0)
    S = Al + np.transpose(np.where(np.tril(np.ones((n, n), bool), -1)[None], Al, 0.0), (0, 2, 1))
    L = np.where(low, _mats(n, L_test), 0.0)
    R = S - L @ np.transpose(L, (0, 2, 1))
    num = np.sqrt((R * R).sum(axis=(1, 2)))
    den = n * np.sqrt((S * S).sum(axis=(1, 2))) * EPS32
    with np.errstate(divide="ignore", invalid="ignore"):
        return np.where(den > 0, num / den, 0.0)


def upper_bits_unchanged(n, before, after):
    """O4 (per matrix): strict upper triangle bitwise identical."""
    b = np.asarray(before, dtype=np.float32).reshape(-1, n, n).view(np.uint32)
    a = np.asarray(after, dtype=np.float32).reshape(-1, n, n).view(np.uint32)
    # canonical flat i + j*n -> reshape gives [b, j, i]; strict upper (i < j)
    # is therefore the strict LOWER triangle of the [j, i] view.
    su = np.tril(np.ones((n, n), bool), -1)[None]
    return np.all(np.where(su, a == b, True), axis=(1, 2))


def accept(n, A_in, L_test, info_test, L64, info64):
    """All of O1-O3 per matrix; returns dict of per-matrix arrays + ok mask.
    ``strict`` is the R10 diagnostic (elementwise relative error on entries
    >= 1e-2 x column max); it is reported and checked separately against
    STRICT_TOL by the parity tests, not folded into ``ok``."""
    info_test = np.asarray(info_test).reshape(-1)
    info64 = np.asarray(info64).reshape(-1)
    o1 = info_test == info64
    e = colnorm_error(n, L_test, L64, info64)
    r = residual(n, A_in, L_test)
    ok_ok = info64 == 0
    o2 = e <= FACTOR_TOL
    o3 = np.where(ok_ok, r <= RESID_TOL, True)
    strict = strict_relative_error(n, L_test, L64, info64)
    return {"info_ok": o1, "err": e, "resid": np.where(ok_ok, r, 0.0), "strict": strict,
            "ok": o1 & o2 & o3}


# ---- solve (SPOTRS / SPOSV) --------------------------------
def solve_residual(n, nrhs, A_in, X, B):
    """Normwise backward error per matrix, FP64:
    max_r ||b_r - A x_r||_inf / ((||A||_inf ||x_r||_inf + ||b_r||_inf) * n * eps32),
    A symmetrised from its FP32 lower triangle.  Acceptance: <= 10."""
    A = _mats(n, A_in)
    low = lower_mask(n)[None]
    Al = np.where(low, A, 0.0)
    S = Al + np.transpose(np.where(np.tril(np.ones((n, n), bool), -1)[None], Al, 0.0), (0, 2, 1))
    Xm = np.asarray(X, dtype=np.float64).reshape(-1, nrhs, n).transpose(0, 2, 1)   # [b, i, r]
    Bm = np.asarray(B, dtype=np.float64).reshape(-1, nrhs, n).transpose(0, 2, 1)
    R = Bm - S @ Xm
    an = np.abs(S).sum(axis=2).max(axis=1)[:, None]                                   # ||A||_inf
    num = np.abs(R).max(axis=1)
    den = (an * np.abs(Xm).max(axis=1) + np.abs(Bm).max(axis=1)) * n * EPS32
    with np.errstate(divide="ignore", invalid="ignore"):
        e = np.where(den > 0, num / den, np.where(num > 0, np.inf, 0.0))
    return e.max(axis=1) if nrhs else np.zeros(len(an))


def solve_forward_error(n, nrhs, X, X64):
    """max_r ||x_r - x64_r||_inf / ||x64_r||_inf per matrix (diagnostic)."""
    Xm = np.asarray(X, dtype=np.float64).reshape(-1, nrhs, n)
    Rm = np.asarray(X64, dtype=np.float64).reshape(-1, nrhs, n)
    num = np.abs(Xm - Rm).max(axis=2)
    den = np.abs(Rm).max(axis=2)
    with np.errstate(divide="ignore", invalid="ignore"):
        e = np.where(den > 0, num / den, num)
    return e.max(axis=1)
