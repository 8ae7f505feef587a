"""CPU checks of the C-ABI boundary: libkde.so loads, exports every symbol
include/kde.h declares, and rejects invalid arguments before touching a GPU."""
import os
import re

import numpy as np
import pytest

import paper_conf_sigmod_heimelkm15_b200 as K

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "kde.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(kde_[a-z_0-9]+)\s*\(", txt)))


def test_header_and_binding_agree():
    assert header_symbols() == sorted(K.ABI_SYMBOLS)


def test_library_exports_every_declared_symbol():
    L = K.lib()
    for s in header_symbols():
        assert hasattr(L, s), s
    assert L.kde_abi_version() == 1


def test_status_strings():
    L = K.lib()
    assert L.kde_status_string(0) == b"KDE_OK"
    assert L.kde_status_string(6) == b"KDE_ETRUNC"


@pytest.mark.parametrize("shape,h,msg", [
    ((10, 0), None, "d = 0"),
    ((10, 17), None, "d = 17"),
    ((1, 3), None, "n = 1"),
    ((10, 2), [1.0, 0.0], "h[1]"),
    ((10, 2), [1.0, float("nan")], "h[1]"),
    ((10, 2), [1.0, float("inf")], "h[1]"),
])
def test_create_rejects_invalid_arguments_before_device_work(shape, h, msg):
    with pytest.raises(K.KDEError) as e:
        K.kde_create(np.zeros(shape, np.float32), h)
    assert e.value.status == K.KDE_EINVAL
    assert msg in str(e.value)


def test_null_model_is_rejected():
    import ctypes
    L = K.lib()
    h = np.zeros(2)
    assert L.kde_get_bandwidth(None, h.ctypes.data_as(ctypes.c_void_p)) == K.KDE_EINVAL
    assert L.kde_synchronize(None) == K.KDE_EINVAL
    K.kde_destroy(None)  # no-op


def test_shard_ranges_cover_rows_exactly():
    from paper_conf_sigmod_heimelkm15_b200.dist import shard_range
    for n in (2, 7, 1000, 2**20 + 3):
        for w in (1, 2, 3, 8):
            spans = [shard_range(n, r, w) for r in range(w)]
            assert spans[0][0] == 0
            for (o1, n1), (o2, _) in zip(spans, spans[1:]):
                assert o1 + n1 == o2
            assert spans[-1][0] + spans[-1][1] == n
            assert max(s[1] for s in spans) - min(s[1] for s in spans) <= 1
