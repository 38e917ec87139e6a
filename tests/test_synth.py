"""The seeded generators (synth/) produce what DESIGN.md's input recipe says."""
import numpy as np
import pytest

import synth


def mat(n, flat):
    return np.asarray(flat).reshape(-1, n, n).transpose(0, 2, 1)


def test_mix64_known_values():
    # splitmix64 finaliser reference values: mix64(0) == 0 and the classic
    # splitmix64 stream seeded with 0 (state += golden gamma, then mix).
    assert int(synth.mix64(np.uint64(0))) == 0
    g = 0x9E3779B97F4A7C15
    outs = [int(synth.mix64(np.uint64((g * k) % 2**64))) for k in (1, 2, 3)]
    assert outs == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


@pytest.mark.parametrize("kind", synth.KINDS)
@pytest.mark.parametrize("n", [1, 2, 8, 16, 32, 64])
def test_generators_spd_exact_symmetric(kind, n):
    b = np.arange(0, 600, 7, dtype=np.uint64)
    A = synth.generate(n, kind, 2017, b, upper="mirror")
    M = mat(n, A).astype(np.float64)
    assert np.array_equal(M, M.transpose(0, 2, 1))
    if kind == "l0":
        # SPD by construction: exactly L0 L0^T with a positive diagonal L0
        # (L0 is badly conditioned at large n, so no eigenvalue test here)
        L0 = synth.l0_factor(n, 2017, b)
        assert np.array_equal(M, L0 @ L0.transpose(0, 2, 1))
        assert (np.diagonal(L0, axis1=1, axis2=2) > 0).all()
        return
    ev = np.linalg.eigvalsh(M)
    assert (ev > 0).all()
    if kind == "dd":
        assert ev.min() > 1.0 - 1e-9 and ev.max() < 2 * n + 1
        assert (np.abs(np.tril(M, -1)) <= 1).all()


def test_partition_invariance():
    n = 9
    full = synth.generate(n, "als", 5, np.arange(100, dtype=np.uint64))
    part = np.concatenate([synth.generate(n, "als", 5, np.arange(s, s + 25, dtype=np.uint64))
                           for s in range(0, 100, 25)])
    assert np.array_equal(full.view(np.uint32), part.view(np.uint32))


def test_upper_modes():
    n = 5
    b = np.arange(4, dtype=np.uint64)
    An = synth.generate(n, "dd", 1, b, upper="nan")
    Az = synth.generate(n, "dd", 1, b, upper="zero")
    su = np.triu(np.ones((n, n), bool), 1)
    Mn = mat(n, An.view(np.uint32))
    assert (Mn[:, su] == synth.UPPER_NAN_BITS).all()
    assert (mat(n, Az)[:, su] == 0).all()
    assert np.array_equal(mat(n, An)[:, ~su], mat(n, Az)[:, ~su])


def test_fail_plan_and_count():
    n, seed_f, P = 32, 2018, 17
    b = np.arange(5000, dtype=np.uint64)
    f, kk = synth.fail_plan(n, seed_f, P, b)
    assert abs(f.mean() - 1 / P) < 0.02
    assert ((kk >= 0) & (kk < n)).all()
    assert synth.expected_fail_count(n, seed_f, P, 0, 5000, block=999) == int(f.sum())
    A = synth.generate(n, "dd", 1, b[:300], fail_seed=seed_f, fail_period=P)
    M = mat(n, A)
    for t in np.nonzero(f[:300])[0]:
        assert M[t, kk[t], kk[t]] == -1.0


def test_als_rank_structure():
    n = 16
    b = np.arange(50, dtype=np.uint64)
    kb = 1 + (synth.hash3(3, b, synth.E_KB) % np.uint64(2 * n)).astype(int)
    M = mat(n, synth.generate(n, "als", 3, b)).astype(np.float64)
    for t in range(50):
        reg = kb[t] / 16.0
        ev = np.linalg.eigvalsh(M[t])
        # Y^T Y has rank <= k_b, so at least n - k_b eigenvalues equal the regulariser
        assert (np.abs(ev - reg) < 1e-9).sum() >= max(0, n - kb[t])


def test_rhs_generator_exact_and_partition_invariant():
    n, nrhs = 7, 3
    B = synth.generate_rhs(n, nrhs, 5, np.arange(100, dtype=np.uint64))
    assert B.shape == (100, n * nrhs) and B.dtype == np.float32
    assert np.array_equal(B.astype(np.float64) * 4096, np.round(B.astype(np.float64) * 4096))
    assert B.min() >= -8 and B.max() < 8
    part = np.concatenate([synth.generate_rhs(n, nrhs, 5, np.arange(s, s + 50, dtype=np.uint64))
                           for s in (0, 50)])
    assert np.array_equal(B.view(np.uint32), part.view(np.uint32))
