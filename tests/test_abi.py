"""The C-ABI library loads, exports every symbol include/*.h declares, and its
host-side argument checks / quick returns behave as the header documents.
No compute call is made (these run without a GPU)."""
import ctypes
import glob
import os
import re

import pytest

import paper_conf_ipps_gatesklpd17_b200 as bsp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    if not os.path.exists(bsp.LIB_PATH):
        from paper_conf_ipps_gatesklpd17_b200 import build
        build.build()
    return bsp.lib()


def header_functions():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        txt = open(h).read()
        txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
        for m in re.finditer(r"^\s*(?:int|int64_t|void)\s+\**(\w+)\s*\(", txt, flags=re.M):
            names.add(m.group(1))
    return names


def test_every_header_symbol_is_exported(L):
    names = header_functions()
    assert len(names) >= 11
    for n in names:
        assert hasattr(L, n), n
    assert set(bsp.EXPORTS) == names


def test_version_and_sizes(L):
    assert bsp.bspotrf_version() >= 10000
    assert bsp.batch_interleaved_elems(3, 70, 32) == 96 * 9
    assert bsp.batch_interleaved_elems(3, 70, 0) == 70 * 9
    assert bsp.batch_interleaved_elems(0, 70, 32) == 0
    assert bsp.batch_interleaved_elems(5, 0, 64) == 0
    assert bsp.batch_interleaved_elems(64, 1 << 25, 32) == (1 << 25) * 4096
    assert L.batch_interleaved_elems(3, 70, 33) == -1
    assert L.batch_interleaved_elems(65, 70, 32) == -1
    assert L.batch_interleaved_elems(3, -1, 32) == -1
    assert bsp.batch_spotrf_host_bytes(16, 1000, 32) == 4 * 136 * 1000


def test_argument_errors_enqueue_nothing(L):
    f = L.batch_spotrf_interleaved
    fake = 0x1000   # never dereferenced: every call below fails its checks first
    assert f(-1, 10, 32, fake, fake, None) == -1
    assert f(65, 10, 32, fake, fake, None) == -1
    assert f(4, -1, 32, fake, fake, None) == -2
    assert f(4, 10, 31, fake, fake, None) == -3
    assert f(4, 10, -32, fake, fake, None) == -3
    assert f(4, 10, 32, None, fake, None) == -4
    assert f(4, 10, 32, fake + 4, fake, None) == -4       # not 16-B aligned
    assert f(4, 10, 32, fake, None, None) == -5
    # quick returns: nothing touched, success
    assert f(0, 10, 32, None, None, None) == 0
    assert f(4, 0, 32, None, None, None) == 0
    g = L.batch_canonical_to_interleaved
    assert g(4, 10, 32, None, fake, None) == -4
    assert g(4, 10, 32, fake, None, None) == -5
    assert g(4, 10, 32, fake, fake + 64, None) == -5      # overlapping
    assert g(4, 10, 7, fake, fake, None) == -3
    h = L.batch_spotrf_interleaved_host
    assert h(4, 10, 32, fake, fake, None, -1, None) == -6
    assert h(4, 10, 32, None, fake, None, 0, None) == -4
    nf = ctypes.c_int32(99)
    assert h(0, 10, 32, None, None, ctypes.addressof(nf), 0, None) == 0 and nf.value == 0
    c = L.batch_spotrf_canonical
    assert c(-1, 10, fake, fake, None, None) == -1
    assert c(21, 10, fake, fake, None, None) == -1       # BSPOTRF_CANON_MAX_N = 20
    assert c(4, -1, fake, fake, None, None) == -2
    assert c(4, 10, None, fake, None, None) == -3
    assert c(4, 10, fake + 2, fake, None, None) == -3    # not 4-B aligned
    assert c(4, 10, fake, None, None, None) == -4
    assert c(0, 10, None, None, None, None) == 0 and c(4, 0, None, None, None, None) == 0
    s = L.bspotrf_synth_generate
    assert s(4, 10, 32, 0, 7, 1, 0, 0, 0, fake, None) == -5
    assert s(4, 10, 32, 0, 0, 1, 9, 0, 0, fake, None) == -6


def test_tuning_table_covers_every_n(L):
    for n in range(1, 65):
        for chunk in (0, 32, 64):
            t = bsp.bspotrf_get_tuning(n, chunk)
            assert t.variant in (bsp.VARIANT_REG, bsp.VARIANT_SMEM, bsp.VARIANT_TILE,
                                 bsp.VARIANT_PANEL, bsp.VARIANT_PTMEM, bsp.VARIANT_RTMA,
                                 bsp.VARIANT_RTMAP, bsp.VARIANT_QTM, bsp.VARIANT_REGX,
                                 bsp.VARIANT_RCW, bsp.VARIANT_REGV, bsp.VARIANT_RCW16, bsp.VARIANT_RCWD,
                                 bsp.VARIANT_RCWP)
            assert t.threads_per_block % 32 == 0
    with pytest.raises(bsp.BspotrfError):
        bsp.bspotrf_get_tuning(65, 32)


def test_explicit_tuning_rejects_unavailable(L):
    t = bsp.Tuning(bsp.VARIANT_REG, 128, 0, 0)
    fake = 0x1000
    # REG is not instantiated past n = 24: -7 before any launch
    assert L.batch_spotrf_interleaved_ex(40, 10, 32, fake, fake, None, ctypes.byref(t), None) == -7
    t = bsp.Tuning(bsp.VARIANT_SMEM, 32, 14, 1)   # TMA staging needs chunk in {32,64,128}
    assert L.batch_spotrf_interleaved_ex(28, 10, 0, fake, fake, None, ctypes.byref(t), None) == -7
    t = bsp.Tuning(bsp.VARIANT_PTMEM, 128, 16, 1)  # PTMEM TMA staging needs chunk 32
    assert L.batch_spotrf_interleaved_ex(32, 10, 64, fake, fake, None, ctypes.byref(t), None) == -7
    t = bsp.Tuning(bsp.VARIANT_PTMEM, 128, 16, 2)  # not instantiated below n = 24
    assert L.batch_spotrf_interleaved_ex(20, 10, 32, fake, fake, None, ctypes.byref(t), None) == -7
    t = bsp.Tuning(bsp.VARIANT_REG, 48, 0, 0)     # tpb not a multiple of 32
    assert L.batch_spotrf_interleaved_ex(8, 10, 32, fake, fake, None, ctypes.byref(t), None) == -7
    t = bsp.Tuning(bsp.VARIANT_REG, 128, 0, 0, 101)   # carveout outside 0..100 percent
    assert L.batch_spotrf_interleaved_ex(8, 10, 32, fake, fake, None, ctypes.byref(t), None) == -7
    t = bsp.Tuning(bsp.VARIANT_REG, 128, 0, 0, -1)
    assert L.batch_spotrf_interleaved_ex(8, 10, 32, fake, fake, None, ctypes.byref(t), None) == -7


def test_tuning_struct_matches_header():
    """bspotrf_tuning in include/bspotrf.h: five ints, carveout last (Table I's
    L1/shared parameter); the table's rows all use the driver default or a
    percentage."""
    hdr = open(os.path.join(ROOT, "include", "bspotrf.h")).read()
    body = hdr[hdr.index("typedef struct {", hdr.index("Launch tuning")):hdr.index("} bspotrf_tuning;")]
    fields = re.findall(r"^\s*int\s+(\w+);", body, flags=re.M)
    assert fields == [f for f, _ in bsp.Tuning._fields_] == \
        ["variant", "threads_per_block", "param", "staging", "carveout"]
    for n in range(1, 65):
        for chunk in (0, 32, 64, 96):
            assert 0 <= bsp.bspotrf_get_tuning(n, chunk).carveout <= 100


def test_product_never_imports_oracle():
    """The product path must not route through oracle/ (or any CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_gatesklpd17_b200")
    for f in glob.glob(os.path.join(pkg, "**", "*.py"), recursive=True) + \
            glob.glob(os.path.join(pkg, "csrc", "**", "*.*"), recursive=True):
        txt = open(f, errors="ignore").read()
        assert not re.search(r"^\s*(from|import)\s+oracle", txt, flags=re.M), f
        assert "liboracle" not in txt and "oracle/" not in txt.replace("oracle/ (", ""), f
    for f in glob.glob(os.path.join(ROOT, "oracle", "*.*")):
        txt = open(f, errors="ignore").read()
        assert "paper_conf_ipps_gatesklpd17_b200" not in txt.replace(
            "paper_conf_ipps_gatesklpd17_b200/csrc", "").replace(
            "(``paper_conf_ipps_gatesklpd17_b200``)", ""), f


def test_every_table_choice_is_built():
    """The default (core) build must hold the instance of every tuning-table
    row it can reach, for every n and chunk class (host logic, no GPU)."""
    for n in range(1, 65):
        for chunk in (0, 32, 64, 96, 128, 256, 512, 1024):
            t = bsp.bspotrf_get_tuning(n, chunk)
            assert bsp.bspotrf_tuning_available(n, chunk, t), (n, chunk, t.as_dict())
    # an explicit tuning with no instance is reported, not launched
    assert not bsp.bspotrf_tuning_available(40, 32, dict(variant=bsp.VARIANT_REG, threads_per_block=128,
                                                         param=0, staging=0))
    with pytest.raises(bsp.BspotrfError):
        bsp.bspotrf_tuning_available(65, 32, dict(variant=1, threads_per_block=0, param=0, staging=0))
