"""CPU oracle for batched Cholesky on (chunked-)interleaved storage.

TEST INFRASTRUCTURE.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product (``paper_conf_ipps_gatesklpd17_b200``) never imports it,
and it never imports the product: the two share no code.  The only common
dependency is ``synth`` (seeded input generators, no method arithmetic).

Contents
--------
* ``potrf``            -- FP64 Algorithm 1 over a canonical
                          batch; C in ``cholesky.c`` (see its header).
* ``potrs``            -- FP64 forward/backward substitution.
* ``spotrf_fig9_fp32`` -- FP32 op-order emulator of Fig. 9 (debugging aid).
* ``layout``           -- the interleaved address formula (PAPER.md:130-153,
                          222-231) and plain (de)interleaving by that formula.
* ``checks``           -- the acceptance metrics O1-O4.
* ``metrics``          -- flop and byte models.

Pin map (what fixes each function other than itself; ``-m "not gpu"``):

* ``potrf``             hand-worked 2x2/3x3/4x4 (golden/handworked_p1.json),
                        integer L0 exactness, identity/diagonal, tridiagonal
                        Toeplitz closed forms, info = k, LAPACK dpotrf
                        (tests/test_oracle_pins.py)
* ``potrs``             hand-worked systems (golden/handworked_solve_p11.json),
                        integer systems, LAPACK dpotrs (tests/test_oracle_solve.py)
* ``layout.offset`` / ``to_/from_interleaved``  Fig. 10 pointer walks replayed,
                        hand-built layouts (tests/test_oracle_layout.py)
* ``layout.rect_*``     hand-worked offsets and a value-naming scatter,
                        square case == the matrix formula (test_oracle_layout.py)
* ``checks.residual`` / ``solve_residual`` / ``strict_relative_error`` /
  ``colnorm_error``     closed-form values of hand-perturbed 2x2/3x3 factors and
                        solutions, so a dropped n, eps = 2^-24, a wrong norm or a
                        transposed right-hand-side index changes the number
                        (tests/test_oracle_checks.py)
* ``metrics``           the SURVEY table's per-n numbers (test_oracle_checks.py)
* ``spotrf_fig9_fp32``  debugging aid; integer-L0 exactness only.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cholesky.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile cholesky.c -> liboracle.so (plain C, -O2, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11", "-fPIC",
               "-shared", "-pthread", _SRC, "-o", _LIB + ".tmp", "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            lib.oracle_potrf_batch.restype = ctypes.c_int
            lib.oracle_potrf_batch.argtypes = [
                ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p,
                ctypes.c_void_p, ctypes.c_int]
            lib.oracle_potrs_batch.restype = ctypes.c_int
            lib.oracle_potrs_batch.argtypes = [
                ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p,
                ctypes.c_void_p]
            lib.oracle_spotrf_fig9_fp32_batch.restype = ctypes.c_int
            lib.oracle_spotrf_fig9_fp32_batch.argtypes = [
                ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
            _lib = lib
    return _lib


def default_threads() -> int:
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def potrf(n: int, A, nthreads: int | None = None):
    """FP64 oracle factor of a canonical FP32 batch.

    A: array-like (batch, n*n) or (batch, n, n) float32, canonical column-major
    per matrix (element (i, j) at flat index i + j*n).  Only i >= j is read.
    Returns (L, info): L float64 (batch, n*n) canonical (strict upper 0),
    info int32 (batch,).
    """
    A = np.asarray(A, dtype=np.float32)
    B = A.shape[0] if A.ndim > 1 else (A.size // (n * n) if n else 0)
    A = np.ascontiguousarray(A.reshape(B, n * n))
    L = np.zeros((B, n * n), dtype=np.float64)
    info = np.zeros(B, dtype=np.int32)
    if B == 0 or n == 0:
        return L, info
    lib = _load()
    rc = lib.oracle_potrf_batch(n, B, A.ctypes.data, L.ctypes.data, info.ctypes.data,
                                nthreads or default_threads())
    if rc != 0:
        raise RuntimeError(f"oracle_potrf_batch failed rc={rc}")
    return L, info


def potrs(n: int, nrhs: int, L64, B):
    """FP64 forward + backward substitution with the oracle
    factor L64 (batch, n*n) float64 and canonical FP32 right-hand sides B
    (batch, n*nrhs), element (i, r) at i + r*n.  Returns X float64 (batch, n*nrhs)."""
    L64 = np.ascontiguousarray(np.asarray(L64, dtype=np.float64).reshape(-1, n * n))
    B = np.ascontiguousarray(np.asarray(B, dtype=np.float32).reshape(-1, n * nrhs))
    X = np.zeros(B.shape, dtype=np.float64)
    if B.shape[0] and n and nrhs:
        rc = _load().oracle_potrs_batch(n, nrhs, B.shape[0], L64.ctypes.data, B.ctypes.data,
                                        X.ctypes.data)
        if rc != 0:
            raise RuntimeError("oracle_potrs_batch failed")
    return X


def spotrf_fig9_fp32(n: int, A):
    """FP32 emulation of Fig. 9's op order (debugging aid; not the oracle)."""
    A = np.ascontiguousarray(np.asarray(A, dtype=np.float32).reshape(-1, n * n))
    B = A.shape[0]
    W = np.zeros((B, n * n), dtype=np.float32)
    info = np.zeros(B, dtype=np.int32)
    if B and n:
        _load().oracle_spotrf_fig9_fp32_batch(n, B, A.ctypes.data, W.ctypes.data,
                                              info.ctypes.data)
    return W, info


from . import checks, layout, metrics  # noqa: E402,F401
