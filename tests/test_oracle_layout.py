"""Pins of the oracle's layout definition (oracle/layout.py) -- pin P9.

The paper fixes the interleaved address only through Fig. 10's pointer walks
 and the prose of Sec. II.B.  These tests
replay the walks literally and brute-force small cases by hand.
"""
import numpy as np
import pytest

from oracle import layout


@pytest.mark.parametrize("N", [1, 2, 5, 8, 16, 32])
def test_fig10_load_lower_walk_matches_formula(N):
    """NB = N: load_lower visits exactly the lower triangle at (i + j*N)*32."""
    walk = layout.fig10_load_lower_walk(N, N)
    assert len(walk) == N * (N + 1) // 2
    for off, m, n in walk:
        assert m >= n
        assert off == layout.offset(N, 10**6, 32, 0, m, n)
    # lane l of the chunk: the same walk shifted by l
    off0 = np.array([w[0] for w in walk])
    for lane in (1, 17, 31):
        offs = [layout.offset(N, 10**6, 32, lane, m, n) for _, m, n in walk]
        assert np.array_equal(np.array(offs), off0 + lane)


@pytest.mark.parametrize("N,NB", [(8, 2), (8, 4), (12, 3), (16, 8)])
def test_fig10_tile_walks_match_formula(N, NB):
    for _m in range(N // NB):
        for _n in range(_m + 1):
            for off, m, n in layout.fig10_load_full_walk(N, NB, _m, _n):
                assert off == layout.offset(N, 10**6, 32, 0, _m * NB + m, _n * NB + n)
        for off, m, n in layout.fig10_load_lower_walk(N, NB, _m, _m):
            assert off == layout.offset(N, 10**6, 32, 0, _m * NB + m, _m * NB + n)


def test_handworked_small_layouts():
    # n = 2, batch = 3, simple interleaved (chunk 0 -> C = 3):
    # memory = [a00 of m0, m1, m2 | a10 of m0, m1, m2 | a01 ... | a11 ...]
    canon = np.array([[0, 1, 2, 3], [10, 11, 12, 13], [20, 21, 22, 23]], np.float32)
    got = layout.to_interleaved(2, 0, canon)
    assert got.tolist() == [0, 10, 20, 1, 11, 21, 2, 12, 22, 3, 13, 23]
    # chunk 32 with batch 3: one chunk of 32 lanes, lanes 3..31 are pad
    got = layout.to_interleaved(2, 32, canon, fill_bits=0x7F800001)
    assert got.size == 32 * 4
    for e in range(4):
        assert got[e * 32:e * 32 + 3].tolist() == [canon[0, e], canon[1, e], canon[2, e]]
        assert (got[e * 32 + 3:(e + 1) * 32].view(np.uint32) == 0x7F800001).all()


@pytest.mark.parametrize("n,batch,chunk", [(1, 1, 32), (3, 70, 32), (3, 70, 64), (4, 33, 0),
                                           (5, 129, 128), (2, 512, 512), (7, 1000, 96)])
def test_bijection_and_roundtrip(n, batch, chunk):
    rng = np.random.default_rng(0)
    canon = rng.standard_normal((batch, n * n)).astype(np.float32)
    inter = layout.to_interleaved(n, chunk, canon)
    C = layout.chunk_of(batch, chunk)
    assert inter.size == -(-batch // C) * C * n * n
    back = layout.from_interleaved(n, batch, chunk, inter)
    assert np.array_equal(back.view(np.uint32), canon.view(np.uint32))
    b = np.arange(batch)[:, None]
    e = np.arange(n * n)[None, :]
    offs = layout.offset(n, batch, chunk, b, e % n, e // n).ravel()
    assert np.unique(offs).size == offs.size and offs.min() >= 0 and offs.max() < inter.size
    assert layout.pad_lane_offsets(n, batch, chunk).size == inter.size - batch * n * n


def test_chunks_are_contiguous_and_coalesced():
    """each chunk occupies a contiguous region; the
    same (i, j) of consecutive matrices are consecutive (one 128-B line per 32)."""
    n, C = 6, 64
    for b in range(0, 256, 37):
        for i in range(n):
            for j in range(i + 1):
                o = layout.offset(n, 256, C, b, i, j)
                assert (b // C) * C * n * n <= o < (b // C + 1) * C * n * n
                if b % C != C - 1:
                    assert layout.offset(n, 256, C, b + 1, i, j) == o + 1


# ---- right-hand-side (rectangular) layout, SURVEY §8(f) f1 -----------------
# The n x nrhs block of matrix b is interleaved like the matrices (same chunk C):
# element (i, r) at (b // C) * C * n * nrhs + (i + r * n) * C + b % C
# (include/bspotrf.h, "Solves").  Offsets below are worked out by hand.

def test_rect_offset_handworked():
    # rows = 3, cols = 2, batch = 40, chunk 32: two chunks of 32 * 6 floats.
    assert layout.rect_storage_elems(3, 2, 40, 32) == 2 * 32 * 6 == 384
    assert layout.rect_offset(3, 2, 40, 32, 0, 0, 0) == 0
    assert layout.rect_offset(3, 2, 40, 32, 5, 2, 0) == 2 * 32 + 5 == 69
    assert layout.rect_offset(3, 2, 40, 32, 5, 0, 1) == 3 * 32 + 5 == 101
    assert layout.rect_offset(3, 2, 40, 32, 33, 2, 1) == 192 + 5 * 32 + 1 == 353
    # chunk 0: C = batch = 40, one chunk
    assert layout.rect_storage_elems(3, 2, 40, 0) == 240
    assert layout.rect_offset(3, 2, 40, 0, 33, 2, 1) == 5 * 40 + 33 == 233
    assert layout.rect_offset(3, 2, 40, 0, 39, 0, 1) == 3 * 40 + 39 == 159
    # cols = 1 (one right-hand side): a vector per matrix
    assert layout.rect_offset(4, 1, 100, 64, 70, 3, 0) == 64 * 4 + 3 * 64 + 6 == 454
    # empty problems
    assert layout.rect_storage_elems(0, 2, 5, 32) == 0
    assert layout.rect_storage_elems(3, 0, 5, 32) == 0
    assert layout.rect_storage_elems(3, 2, 0, 32) == 0


def test_rect_scatter_gather_handworked():
    rows, cols, batch, chunk = 3, 2, 40, 32
    b = np.arange(batch)[:, None]
    e = np.arange(rows * cols)[None, :]
    i, r = e % rows, e // rows
    canon = (1000 * b + 10 * i + r).astype(np.float32)      # value names its (b, i, r)
    out = layout.rect_to_interleaved(rows, cols, chunk, canon, fill_bits=0x7FC0DEAD)
    assert out.size == 384
    assert out[69] == 5020 and out[101] == 5001 and out[353] == 33021 and out[0] == 0
    # pad lanes: matrices 40..63 of the second chunk, every element
    for ee in range(6):
        blk = out[192 + ee * 32 + 8:192 + (ee + 1) * 32]
        assert (blk.view(np.uint32) == 0x7FC0DEAD).all()
    assert (out.view(np.uint32) == 0x7FC0DEAD).sum() == 24 * 6
    back = layout.rect_from_interleaved(rows, cols, batch, chunk, out)
    assert np.array_equal(back, canon)
    # a transposed (i, r) reading would put (b=5, i=0, r=1) at 1*32+5: it must not
    assert out[1 * 32 + 5] == 5010


@pytest.mark.parametrize("n,batch,chunk", [(5, 77, 32), (16, 70, 64), (3, 33, 0)])
def test_rect_square_equals_matrix_layout(n, batch, chunk):
    """rows == cols reduces to the matrix formula pinned by Fig. 10's walks."""
    b = np.arange(batch)[:, None]
    e = np.arange(n * n)[None, :]
    assert np.array_equal(layout.rect_offset(n, n, batch, chunk, b, e % n, e // n),
                          layout.offset(n, batch, chunk, b, e % n, e // n))
