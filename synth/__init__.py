"""Seeded synthetic SPD batches: the counter-based input generator (host side).

This module is the ONE thing the oracle (``oracle/``) and the CUDA path share,
and it holds none of the method's arithmetic (no square roots, no scaling, no
rank-1 updates): it only draws integers from a counter hash and assembles
exactly-representable FP32 inputs.  The CUDA library implements the *same*
counter-based generator independently (``csrc/synth.cu``); the GPU tests check
the two bit for bit.

Hash (both sides):  splitmix64 finaliser ``mix64`` and

    h(seed, b, e) = mix64( mix64(seed * G + b) ^ (e * K1 + K2) )

with ``b`` the *global* matrix index (so any GPU count / partition produces the
same matrices) and ``e`` an element/stream counter.  Element (i, j), i >= j, of
matrix b uses e = i + j*n (canonical column-major index).

Generators (recipes stated in DESIGN.md "Input recipe"):

* ``dd``  diagonally dominant SPD.  a_ij = (u24 - 2^23) / 2^23 in [-1, 1) for
  i > j (u24 = h >> 40), a_ii = n + (h >> 48) / 2^16.  Every value is exact in
  FP32; by Gershgorin every eigenvalue lies in (1, 2n + 1).
* ``als`` ALS-shaped regularised Gram matrix (the workload PAPER.md:22-24
  motivates; parameters are our reading R16 in DESIGN.md).  k_b = 1 + h mod 2n
  "ratings", Y in {-256..255}/256 of shape k_b x n, A = Y^T Y + (k_b/16) I.
  Y[r, c] = (fmix32(key_b ^ ((r*n + c) * 0x9E3779B1 mod 2^32)) >> 23) - 256
  with key_b the low 32 bits of h(seed, b, E_Y) and fmix32 MurmurHash3's
  32-bit finaliser (cheap enough to recompute on the GPU).
  All partial sums are multiples of 2^-16 below 2^8, so A is exact in FP32 for
  any summation order.
* ``l0``  integer factor (pin P2): L0 strictly-lower in {-3..3}, diag in
  {1, 2, 4}, A = L0 L0^T (exact integers).  ``l0_factor`` returns L0 itself.

Failure injection (pin P5/P10): matrices b with ``hf % P == 0``,
hf = h(seed_f, b, E_FAIL), get pivot kk = (hf >> 32) % n forced negative:
a_kk = -1 (dd/als), or a_kk = sum_{j<kk} L0_kj^2 - 1 (l0: Schur pivot exactly -1).
Every earlier pivot is unchanged, so LAPACK-style info = kk + 1.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "mix64", "fmix32", "hash3", "generate", "l0_factor", "fail_plan", "expected_fail_count",
    "UPPER_NAN_BITS", "PAD_BITS", "KINDS",
]

_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_G = np.uint64(0x9E3779B97F4A7C15)
_K1 = np.uint64(0xD1B54A32D192ED03)
_K2 = np.uint64(0x632BE59BD9B4E019)

# Stream counters kept far above any element index (n <= 64 -> e < 4096).
E_KB = 1 << 20        # ALS: number of ratings k_b
E_Y = 1 << 21         # ALS: Y[r, c] uses E_Y + r*n + c
E_FAIL = 1 << 22      # failure injection draw

# Bit patterns: strict-upper sentinel (quiet NaN with payload) for parity runs,
# and the pad-lane sentinel written around the batch by tests.
UPPER_NAN_BITS = 0x7FC0FFEE
PAD_BITS = 0xFFC0DEAD

KINDS = ("dd", "als", "l0")
E_RHS = 1 << 23       # right-hand sides: B[i, r] uses E_RHS + i + r*n


def mix64(z):
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def fmix32(x):
    """MurmurHash3 32-bit finaliser on uint32 arrays (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint32)
    with np.errstate(over="ignore"):
        x = x ^ (x >> np.uint32(16))
        x = x * np.uint32(0x85EBCA6B)
        x = x ^ (x >> np.uint32(13))
        x = x * np.uint32(0xC2B2AE35)
        x = x ^ (x >> np.uint32(16))
    return x


def hash3(seed, b, e):
    """h(seed, b, e) as defined in the module docstring (broadcasting)."""
    seed = np.asarray(seed, dtype=np.uint64)
    b = np.asarray(b, dtype=np.uint64)
    e = np.asarray(e, dtype=np.uint64)
    with np.errstate(over="ignore"):
        hb = mix64(seed * _G + b)
        return mix64(hb ^ (e * _K1 + _K2))


def _lower_pairs(n):
    i, j = np.tril_indices(n)          # i >= j
    return i, j


def _l0_entries(n, seed, b):
    """Integer L0 (len(b), n, n), lower triangular, as int64."""
    B = b.shape[0]
    i, j = _lower_pairs(n)
    e = (i + j * n).astype(np.uint64)
    h = hash3(seed, b[:, None], e[None, :])
    L = np.zeros((B, n, n), dtype=np.int64)
    off = (h % np.uint64(7)).astype(np.int64) - 3
    dg = np.array([1, 2, 4], dtype=np.int64)[(h % np.uint64(3)).astype(np.int64)]
    vals = np.where((i == j)[None, :], dg, off)
    L[:, i, j] = vals
    return L


def l0_factor(n, seed, b):
    """The exact integer factor L0 of the ``l0`` generator, float64 (len(b), n, n)."""
    b = np.atleast_1d(np.asarray(b, dtype=np.uint64))
    return _l0_entries(n, seed, b).astype(np.float64)


def fail_plan(n, seed_f, period, b):
    """For global indices b: (is_failed bool array, kk 0-based pivot index)."""
    b = np.atleast_1d(np.asarray(b, dtype=np.uint64))
    if period <= 0 or n == 0:
        return np.zeros(b.shape, bool), np.zeros(b.shape, np.int64)
    hf = hash3(seed_f, b, E_FAIL)
    failed = (hf % np.uint64(period)) == 0
    kk = ((hf >> np.uint64(32)) % np.uint64(n)).astype(np.int64)
    return failed, kk


def expected_fail_count(n, seed_f, period, b_begin, b_end, block=1 << 22):
    """Number of injected failures among global indices [b_begin, b_end)."""
    total = 0
    for s in range(b_begin, b_end, block):
        b = np.arange(s, min(b_end, s + block), dtype=np.uint64)
        f, _ = fail_plan(n, seed_f, period, b)
        total += int(f.sum())
    return total


def generate(n, kind, seed, b, upper="mirror", fail_seed=0, fail_period=0):
    """Canonical FP32 batch for global indices ``b``: array (len(b), n*n).

    Element (i, j) of matrix k is at [k, i + j*n] (column-major).
    ``upper``: "mirror" (symmetric), "nan" (UPPER_NAN_BITS sentinel) or "zero".
    """
    b = np.atleast_1d(np.asarray(b, dtype=np.uint64))
    B = b.shape[0]
    out = np.zeros((B, n, n), dtype=np.float32)   # [k, i, j]
    if n == 0 or B == 0:
        return out.reshape(B, n * n)
    i, j = _lower_pairs(n)
    if kind == "dd":
        e = (i + j * n).astype(np.uint64)
        h = hash3(seed, b[:, None], e[None, :])
        off = ((h >> np.uint64(40)).astype(np.int64) - (1 << 23)).astype(np.float64) / float(1 << 23)
        dg = float(n) + (h >> np.uint64(48)).astype(np.float64) / 65536.0
        vals = np.where((i == j)[None, :], dg, off)
        low = vals
    elif kind == "als":
        kb = 1 + (hash3(seed, b, E_KB) % np.uint64(2 * n)).astype(np.int64)
        key = (hash3(seed, b, E_Y) & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        r = np.arange(2 * n)
        c = np.arange(n)
        with np.errstate(over="ignore"):
            ctr = ((r[:, None] * n + c[None, :]).astype(np.uint32) * np.uint32(0x9E3779B1))
        low = np.empty((B, i.shape[0]), dtype=np.float64)
        step = 2048
        for s in range(0, B, step):
            hb = fmix32(key[s:s + step, None, None] ^ ctr[None, :, :])
            Y = (hb >> np.uint32(23)).astype(np.int64) - 256                # (Bs, 2n, n)
            Y = np.where(r[None, :, None] < kb[s:s + step, None, None], Y, 0)
            G = np.einsum("kri,krj->kij", Y, Y)                              # exact int64
            A = G[:, i, j].astype(np.float64) / 65536.0
            A = A + np.where((i == j)[None, :], kb[s:s + step, None] / 16.0, 0.0)
            low[s:s + step] = A
    elif kind == "l0":
        L = _l0_entries(n, seed, b)
        G = np.einsum("kip,kjp->kij", L, L)
        low = G[:, i, j].astype(np.float64)
    else:
        raise ValueError(f"unknown kind {kind!r}")

    if fail_period > 0:
        failed, kk = fail_plan(n, fail_seed, fail_period, b)
        diag_pos = {int(d): int(np.nonzero((i == d) & (j == d))[0][0]) for d in range(n)}
        for k_idx in np.nonzero(failed)[0]:
            d = int(kk[k_idx])
            if kind == "l0":
                L = _l0_entries(n, seed, b[k_idx:k_idx + 1])[0]
                val = float((L[d, :d] ** 2).sum() - 1)
            else:
                val = -1.0
            low[k_idx, diag_pos[d]] = val

    low32 = low.astype(np.float32)
    if not np.array_equal(low32.astype(np.float64), low):
        raise AssertionError("generator value not exactly representable in FP32")
    out[:, i, j] = low32
    if upper == "mirror":
        out[:, j, i] = low32
    elif upper == "nan":
        su, sv = np.triu_indices(n, 1)
        out[:, su, sv] = np.array([UPPER_NAN_BITS], dtype=np.uint32).view(np.float32)[0]
    elif upper != "zero":
        raise ValueError(f"unknown upper mode {upper!r}")
    # canonical column-major: flat index i + j*n  ==  transpose to [k, j, i]
    return np.ascontiguousarray(out.transpose(0, 2, 1)).reshape(B, n * n)


def generate_rhs(n, nrhs, seed, b):
    """Right-hand sides for the solve: canonical (len(b), n*nrhs),
    element (i, r) at i + r*n, values (u16 - 2^15) / 2^12 in [-8, 8) -- exact in FP32."""
    b = np.atleast_1d(np.asarray(b, dtype=np.uint64))
    if n == 0 or nrhs == 0 or b.shape[0] == 0:
        return np.zeros((b.shape[0], n * nrhs), dtype=np.float32)
    e = (E_RHS + np.arange(n * nrhs)).astype(np.uint64)
    h = hash3(seed, b[:, None], e[None, :])
    v = ((h >> np.uint64(48)).astype(np.int64) - (1 << 15)).astype(np.float64) / 4096.0
    return v.astype(np.float32)
