"""Flop and byte models (TEST/BENCH INFRASTRUCTURE; see oracle/__init__.py).

* flops per matrix: n^3/3, "the standard formula ... always used"
  (Sec. III); reading R12 -- not the exact n^3/3 + n^2/2 + n/6.
* algorithmic bytes per matrix for the factorization: the lower triangle read
  once and written once in FP32, plus one int32 info:  4 n (n+1) + 4
  (Fig. 10 load_lower/store_lower).
* layout conversion: the full n x n block read and written: 8 n^2 per matrix.
"""


def flops_per_matrix(n: int) -> float:
    return n ** 3 / 3.0


def factor_bytes_per_matrix(n: int) -> int:
    return 4 * n * (n + 1) + 4


def convert_bytes_per_matrix(n: int) -> int:
    return 8 * n * n
