"""bspotrf-b200: batched FP32 Cholesky (SPOTRF, lower, in place) on the
interleaved / chunked-interleaved layout of Gates et al., IPDPS-W 2017.

Thin Python binding over the C ABI of ``libbspotrf.so`` (include/bspotrf.h,
include/bspotrf_synth.h): the same function names, argument marshalling only.
Every step of the path runs in the library's CUDA kernels; there is no CPU or
PyTorch fallback -- if the library is missing, every call raises.

Tensors are torch tensors (device memory, streams) or raw integer pointers.
"""
from __future__ import annotations

import ctypes
import os
import threading

__all__ = [
    "BspotrfError", "lib", "bspotrf_version", "batch_interleaved_elems",
    "batch_spotrf_interleaved", "batch_spotrf_interleaved_ex", "bspotrf_get_tuning",
    "batch_canonical_to_interleaved", "batch_interleaved_to_canonical", "batch_spotrf_canonical",
    "CANON_MAX_N", "batch_spotrf_interleaved_host", "batch_spotrf_host_bytes",
    "bspotrf_synth_generate", "bspotrf_fill_u32", "bspotrf_probe_copy_lower", "Tuning",
    "batch_interleaved_rhs_elems", "batch_spotrs_interleaved", "batch_sposv_interleaved",
    "bspotrf_tuning_available", "VARIANT_AUTO", "VARIANT_REG", "VARIANT_SMEM", "VARIANT_TILE", "VARIANT_PANEL", "VARIANT_PTMEM", "VARIANT_RTMA", "VARIANT_RTMAP", "VARIANT_QTM", "VARIANT_REGX", "VARIANT_RCW", "VARIANT_REGV", "VARIANT_RCW16", "VARIANT_RCWD", "VARIANT_RCWP",
    "SYNTH_KINDS", "UPPER_MODES", "LIB_PATH",
]

LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libbspotrf.so")

(VARIANT_AUTO, VARIANT_REG, VARIANT_SMEM, VARIANT_TILE, VARIANT_PANEL, VARIANT_PTMEM,
 VARIANT_RTMA, VARIANT_RTMAP, VARIANT_QTM, VARIANT_REGX, VARIANT_RCW, VARIANT_REGV, VARIANT_RCW16,
 VARIANT_RCWD, VARIANT_RCWP) = 0, 1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 11, 12, 13, 14
SYNTH_KINDS = {"dd": 0, "als": 1, "l0": 2}
CANON_MAX_N = 20          # BSPOTRF_CANON_MAX_N
UPPER_MODES = {"mirror": 0, "nan": 1, "keep": 2}

# every exported symbol of include/*.h (checked by tests/test_abi.py)
EXPORTS = (
    "bspotrf_version", "batch_interleaved_elems", "batch_spotrf_interleaved",
    "batch_spotrf_interleaved_ex", "bspotrf_get_tuning", "batch_canonical_to_interleaved",
    "batch_interleaved_to_canonical", "batch_spotrf_interleaved_host", "batch_spotrf_host_bytes",
    "bspotrf_synth_generate", "bspotrf_fill_u32", "bspotrf_probe_copy_lower",
    "batch_interleaved_rhs_elems", "batch_spotrs_interleaved", "batch_sposv_interleaved",
    "bspotrf_tuning_available", "batch_spotrf_canonical",
)


class BspotrfError(RuntimeError):
    """Nonzero return code of a C-ABI call (negative: illegal argument i;
    positive: cudaError_t)."""

    def __init__(self, fn, code):
        self.code = code
        super().__init__(f"{fn} returned {code}")


class Tuning(ctypes.Structure):
    _fields_ = [("variant", ctypes.c_int), ("threads_per_block", ctypes.c_int),
                ("param", ctypes.c_int), ("staging", ctypes.c_int), ("carveout", ctypes.c_int)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_lock = threading.Lock()
_lib = None

_vp, _i32, _i64, _u32, _u64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_uint32, ctypes.c_uint64
_SIGS = {
    "bspotrf_version": (_i32, []),
    "batch_interleaved_elems": (_i64, [_i32, _i64, _i32]),
    "batch_spotrf_interleaved": (_i32, [_i32, _i64, _i32, _vp, _vp, _vp]),
    "batch_spotrf_interleaved_ex": (_i32, [_i32, _i64, _i32, _vp, _vp, _vp, ctypes.POINTER(Tuning), _vp]),
    "bspotrf_get_tuning": (_i32, [_i32, _i32, ctypes.POINTER(Tuning)]),
    "bspotrf_tuning_available": (_i32, [_i32, _i32, ctypes.POINTER(Tuning)]),
    "batch_canonical_to_interleaved": (_i32, [_i32, _i64, _i32, _vp, _vp, _vp]),
    "batch_interleaved_to_canonical": (_i32, [_i32, _i64, _i32, _vp, _vp, _vp]),
    "batch_spotrf_canonical": (_i32, [_i32, _i64, _vp, _vp, _vp, _vp]),
    "batch_spotrf_interleaved_host": (_i32, [_i32, _i64, _i32, _vp, _vp, _vp, _i64, _vp]),
    "batch_spotrf_host_bytes": (_i64, [_i32, _i64, _i32]),
    "bspotrf_synth_generate": (_i32, [_i32, _i64, _i32, _i64, _i32, _u64, _i32, _u64, _i64, _vp, _vp]),
    "bspotrf_fill_u32": (_i32, [_vp, _i64, _u32, _vp]),
    "bspotrf_probe_copy_lower": (_i32, [_i32, _i64, _vp, _vp, _i32, _vp]),
    "batch_interleaved_rhs_elems": (_i64, [_i32, _i32, _i64, _i32]),
    "batch_spotrs_interleaved": (_i32, [_i32, _i32, _i64, _i32, _vp, _vp, _vp]),
    "batch_sposv_interleaved": (_i32, [_i32, _i32, _i64, _i32, _vp, _vp, _vp, _vp, _vp]),
}


def lib():
    """Load libbspotrf.so (fails loudly: there is no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise RuntimeError(
                    f"{LIB_PATH} not built: run `python -m paper_conf_ipps_gatesklpd17_b200.build` "
                    "(there is no CPU fallback)")
            L = ctypes.CDLL(LIB_PATH)
            for name, (res, args) in _SIGS.items():
                fn = getattr(L, name)
                fn.restype = res
                fn.argtypes = args
            _lib = L
    return _lib


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(s):
    if s is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(s, int):
        return s
    return s.cuda_stream


def _check(fn, rc):
    if rc != 0:
        raise BspotrfError(fn, rc)
    return rc


def _need(t, n_elems, dtype_name, what):
    if isinstance(t, int) or t is None:
        return
    if not t.is_contiguous():
        raise ValueError(f"{what} must be contiguous")
    if str(t.dtype) != dtype_name:
        raise ValueError(f"{what} must be {dtype_name}, got {t.dtype}")
    if t.numel() < n_elems:
        raise ValueError(f"{what} has {t.numel()} elements, needs {n_elems}")


def bspotrf_version() -> int:
    return lib().bspotrf_version()


def batch_interleaved_elems(n: int, batch: int, chunk: int) -> int:
    r = lib().batch_interleaved_elems(n, batch, chunk)
    if r < 0:
        raise BspotrfError("batch_interleaved_elems", r)
    return r


def batch_spotrf_host_bytes(n: int, batch: int, chunk: int) -> int:
    return lib().batch_spotrf_host_bytes(n, batch, chunk)


def bspotrf_get_tuning(n: int, chunk: int) -> Tuning:
    t = Tuning()
    _check("bspotrf_get_tuning", lib().bspotrf_get_tuning(n, chunk, ctypes.byref(t)))
    return t


def bspotrf_tuning_available(n: int, chunk: int, tune) -> bool:
    """Whether the library holds a kernel instance for this explicit tuning."""
    if isinstance(tune, dict):
        tune = Tuning(**{k: int(v) for k, v in tune.items()})
    rc = lib().bspotrf_tuning_available(n, chunk, ctypes.byref(tune))
    if rc < 0:
        raise BspotrfError("bspotrf_tuning_available", rc)
    return rc == 1


def batch_spotrf_interleaved(n, batch, chunk, A, info, stream=None):
    """In-place batched SPOTRF (lower) on device interleaved storage A."""
    if n and batch:
        _need(A, batch_interleaved_elems(n, batch, chunk), "torch.float32", "A")
        _need(info, batch, "torch.int32", "info")
    return _check("batch_spotrf_interleaved", lib().batch_spotrf_interleaved(
        n, batch, chunk, _ptr(A), _ptr(info), _stream(stream)))


def batch_spotrf_interleaved_ex(n, batch, chunk, A, info, nfailed=None, tune=None, stream=None):
    """As batch_spotrf_interleaved; nfailed (device int32[1]) is incremented by
    the number of failed matrices; tune: Tuning / dict / None (table)."""
    if n and batch:
        _need(A, batch_interleaved_elems(n, batch, chunk), "torch.float32", "A")
        _need(info, batch, "torch.int32", "info")
        _need(nfailed, 1, "torch.int32", "nfailed")
    tp = None
    if tune is not None:
        if isinstance(tune, dict):
            tune = Tuning(**{k: int(v) for k, v in tune.items()})
        tp = ctypes.byref(tune)
    return _check("batch_spotrf_interleaved_ex", lib().batch_spotrf_interleaved_ex(
        n, batch, chunk, _ptr(A), _ptr(info), _ptr(nfailed), tp, _stream(stream)))


def batch_canonical_to_interleaved(n, batch, chunk, src, dst, stream=None):
    if n and batch:
        _need(src, batch * n * n, "torch.float32", "src")
        _need(dst, batch_interleaved_elems(n, batch, chunk), "torch.float32", "dst")
    return _check("batch_canonical_to_interleaved", lib().batch_canonical_to_interleaved(
        n, batch, chunk, _ptr(src), _ptr(dst), _stream(stream)))


def batch_interleaved_to_canonical(n, batch, chunk, src, dst, stream=None):
    if n and batch:
        _need(src, batch_interleaved_elems(n, batch, chunk), "torch.float32", "src")
        _need(dst, batch * n * n, "torch.float32", "dst")
    return _check("batch_interleaved_to_canonical", lib().batch_interleaved_to_canonical(
        n, batch, chunk, _ptr(src), _ptr(dst), _stream(stream)))


def batch_spotrf_canonical(n, batch, A, info, nfailed=None, stream=None):
    """In-place batched SPOTRF (lower) on device CANONICAL storage A (batch
    consecutive n x n column-major matrices), conversion fused; n <= CANON_MAX_N."""
    if n and batch:
        _need(A, batch * n * n, "torch.float32", "A")
        _need(info, batch, "torch.int32", "info")
        _need(nfailed, 1, "torch.int32", "nfailed")
    return _check("batch_spotrf_canonical", lib().batch_spotrf_canonical(
        n, batch, _ptr(A), _ptr(info), _ptr(nfailed), _stream(stream)))


def batch_spotrf_interleaved_host(n, batch, chunk, hA, hinfo, slab=0, stream=None):
    """End-to-end factorization of HOST interleaved storage (blocking).
    Returns the number of failed matrices."""
    if n and batch:
        _need(hA, batch_interleaved_elems(n, batch, chunk), "torch.float32", "hA")
        _need(hinfo, batch, "torch.int32", "hinfo")
    nf = ctypes.c_int32(0)
    _check("batch_spotrf_interleaved_host", lib().batch_spotrf_interleaved_host(
        n, batch, chunk, _ptr(hA), _ptr(hinfo), ctypes.addressof(nf), slab, _stream(stream)))
    return nf.value


def batch_interleaved_rhs_elems(n: int, nrhs: int, batch: int, chunk: int) -> int:
    r = lib().batch_interleaved_rhs_elems(n, nrhs, batch, chunk)
    if r < 0:
        raise BspotrfError("batch_interleaved_rhs_elems", r)
    return r


def batch_spotrs_interleaved(n, nrhs, batch, chunk, L, B, stream=None):
    """B := A^-1 B with the factor L from batch_spotrf_interleaved (device)."""
    if n and nrhs and batch:
        _need(L, batch_interleaved_elems(n, batch, chunk), "torch.float32", "L")
        _need(B, batch_interleaved_rhs_elems(n, nrhs, batch, chunk), "torch.float32", "B")
    return _check("batch_spotrs_interleaved", lib().batch_spotrs_interleaved(
        n, nrhs, batch, chunk, _ptr(L), _ptr(B), _stream(stream)))


def batch_sposv_interleaved(n, nrhs, batch, chunk, A, B, info, nfailed=None, stream=None):
    """Factor A in place and solve A X = B (fused for n <= 20, nrhs <= 4)."""
    if n and batch:
        _need(A, batch_interleaved_elems(n, batch, chunk), "torch.float32", "A")
        _need(info, batch, "torch.int32", "info")
        if nrhs:
            _need(B, batch_interleaved_rhs_elems(n, nrhs, batch, chunk), "torch.float32", "B")
    return _check("batch_sposv_interleaved", lib().batch_sposv_interleaved(
        n, nrhs, batch, chunk, _ptr(A), _ptr(B), _ptr(info), _ptr(nfailed), _stream(stream)))


def bspotrf_synth_generate(n, batch, chunk, A, kind="dd", seed=2017, b0=0, upper="mirror",
                           fail_seed=0, fail_period=0, stream=None):
    """Fill device interleaved storage A with matrices b0..b0+batch-1 of the
    seeded global sequence (include/bspotrf_synth.h)."""
    if n and batch:
        _need(A, batch_interleaved_elems(n, batch, chunk), "torch.float32", "A")
    return _check("bspotrf_synth_generate", lib().bspotrf_synth_generate(
        n, batch, chunk, b0, SYNTH_KINDS[kind], seed, UPPER_MODES[upper], fail_seed,
        fail_period, _ptr(A), _stream(stream)))


def bspotrf_probe_copy_lower(n, batch, A, info, tpb=128, stream=None):
    """Diagnostic: the REG kernel's memory traffic without arithmetic (chunk 32)."""
    return _check("bspotrf_probe_copy_lower", lib().bspotrf_probe_copy_lower(
        n, batch, _ptr(A), _ptr(info), tpb, _stream(stream)))


def bspotrf_fill_u32(A, value_bits, elems=None, stream=None):
    if elems is None:
        elems = A.numel()
    return _check("bspotrf_fill_u32", lib().bspotrf_fill_u32(_ptr(A), elems, value_bits, _stream(stream)))
