"""C-ABI library checks that need no GPU: it loads, exports every symbol include/czc.h declares,
the Python struct mirrors match the compiled layout, and argument validation fails cleanly."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "czc.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(czc_[a-z_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def czc():
    from paper_conf_cluster_yudgtc21_b200 import build
    build.build()
    import paper_conf_cluster_yudgtc21_b200 as m
    return m


def test_exports_every_declared_symbol(czc):
    names = declared_symbols()
    assert {"czc_init", "czc_assess", "czc_free", "czc_assess_host"} <= set(names)
    lib = ctypes.CDLL(czc.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), f"libczc.so does not export {n}"
    assert set(czc.EXPORTED) == set(names)


def test_struct_layout_and_version(czc):
    assert czc.lib.czc_abi_version() == 5          # v5: czc_config.debug_der (round 2)
    for what, st in ((0, czc.Config), (1, czc.Shape), (2, czc.Result)):
        assert czc.lib.czc_sizeof(what) == ctypes.sizeof(st)
    assert czc.lib.czc_sizeof(7) == 0
    assert 0 < czc.lib.czc_sizeof(3) < 8192
    assert czc.lib.czc_has_nccl() in (0, 1)


def test_strerror(czc):
    for s in range(8):
        assert czc.lib.czc_strerror(s).decode() == czc.STATUS[s]
    assert czc.lib.czc_strerror(99)


def test_validation_without_gpu(czc):
    """Paths that must fail before touching a device."""
    h = ctypes.c_void_p()
    assert czc.lib.czc_init(None, None) == 1                         # NULL out
    bad = czc.make_config(ac_max_lag=czc.MAX_LAG + 1)
    assert czc.lib.czc_init(ctypes.byref(h), ctypes.byref(bad)) == 1
    bad = czc.make_config(ssim_range_mode=3)
    assert czc.lib.czc_init(ctypes.byref(h), ctypes.byref(bad)) == 1
    bad = czc.make_config(pdf_bins=czc.PDF_MAX_BINS + 1)
    assert czc.lib.czc_init(ctypes.byref(h), ctypes.byref(bad)) == 1
    bad = czc.make_config(nranks=2, rank=0)                           # no NCCL uid
    assert czc.lib.czc_init(ctypes.byref(h), ctypes.byref(bad)) == 1
    r = czc.Result()
    shape = czc.make_shape([4, 4, 4])
    assert czc.lib.czc_assess(None, None, None, ctypes.byref(shape), 0, czc.M_ALL, ctypes.byref(r)) == 1
    assert r.computed_mask == 0
    assert czc.lib.czc_assess(None, None, None, ctypes.byref(shape), 0, czc.M_ALL, None) == 1
