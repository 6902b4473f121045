"""C-ABI library checks that need no GPU: the library loads, exports every
function include/medusa.h declares, and rejects bad arguments before touching
the device."""
import ctypes
import os
import re

import pytest

import __graft_entry__ as ge

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "medusa.h")


@pytest.fixture(scope="module")
def lib():
    path = ge.build_medusa()
    return ctypes.CDLL(path)


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(medusa_[a-z_]+)\s*\(", src)))


def test_header_declares_the_three_calls():
    names = _declared()
    for n in ("medusa_materialize", "medusa_kernel_table_set", "medusa_restore"):
        assert n in names


def test_library_exports_every_declared_symbol(lib):
    for n in _declared():
        assert hasattr(lib, n), n


def test_status_strings(lib):
    lib.medusa_status_string.restype = ctypes.c_char_p
    lib.medusa_status_string.argtypes = [ctypes.c_int]
    assert lib.medusa_status_string(0) == b"MEDUSA_OK"
    assert lib.medusa_status_string(-2) == b"MEDUSA_ERR_TRACE"
    assert lib.medusa_status_string(-5) == b"MEDUSA_ERR_CUDA"


def test_argument_errors_need_no_device(lib):
    P, U64, U32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32

    class Slots(ctypes.Structure):
        _fields_ = [("m", P), ("c", P), ("s", P), ("cap", U64)]

    n = U64(7)
    # materialize: null slot table / null output count / oversize trace
    assert lib.medusa_materialize(P(0), U64(0), P(8), U32(0), P(0), P(0), U32(0), None, ctypes.byref(n), P(0)) == -1
    assert n.value == 0
    s = Slots(8, 8, 8, 1)
    assert lib.medusa_materialize(P(0), U64(0), P(8), U32(0), P(0), P(8), U32((1 << 24) + 1), ctypes.byref(s),
                                  ctypes.byref(n), P(0)) == -1
    assert lib.medusa_materialize(P(8), U64(10), P(8), U32(1), P(0), P(0), U32(0), ctypes.byref(s),
                                  ctypes.byref(n), P(0)) == -1  # nodes without times
    assert lib.medusa_materialize(P(12), U64(10), P(8), U32(0), P(0), P(0), U32(0), ctypes.byref(s),
                                  ctypes.byref(n), P(0)) == -1  # misaligned words
    # restore: partial overlap, null report, gather half-specified, n_slots > n_words
    r = P(64)
    assert lib.medusa_restore(P(1024), P(1032), U64(10), ctypes.byref(s), U64(0), P(0), P(0), P(0), U32(0), P(0),
                              P(0), U32(0), r, P(0)) == -1
    assert lib.medusa_restore(P(1024), P(1024), U64(10), ctypes.byref(s), U64(0), P(0), P(0), P(0), U32(0), P(0),
                              P(0), U32(0), P(0), P(0)) == -1
    assert lib.medusa_restore(P(1024), P(1024), U64(10), ctypes.byref(s), U64(0), P(0), P(0), P(0), U32(0), P(64),
                              P(0), U32(3), r, P(0)) == -1
    assert lib.medusa_restore(P(1024), P(1024), U64(10), ctypes.byref(s), U64(11), P(0), P(0), P(0), U32(0), P(0),
                              P(0), U32(0), r, P(0)) == -1
    # kernel table: null with a size
    assert lib.medusa_kernel_table_set(P(0), U32(4), P(0)) == -1
    # buffers plan: null outputs, misaligned trace, captures without array
    np_, nb = U32(5), U64(5)
    assert lib.medusa_buffers_plan(P(8), U32(1), P(0), U32(0), P(0), U64(0), P(8), P(8), P(8), U32(1), None,
                                   ctypes.byref(nb), P(0)) == -1
    assert nb.value == 0
    assert lib.medusa_buffers_plan(P(12), U32(1), P(0), U32(0), P(0), U64(0), P(8), P(8), P(8), U32(1),
                                   ctypes.byref(np_), ctypes.byref(nb), P(0)) == -1
    assert lib.medusa_buffers_plan(P(8), U32(1), P(0), U32(2), P(0), U64(0), P(8), P(8), P(8), U32(1),
                                   ctypes.byref(np_), ctypes.byref(nb), P(0)) == -1
    # save / restore: null report, misaligned blob (16-byte rule), missing replay arrays
    assert lib.medusa_buffers_save(P(8), P(8), U32(1), P(8), U32(1), P(16), P(0), P(0)) == -1
    assert lib.medusa_buffers_save(P(8), P(8), U32(1), P(8), U32(1), P(24), P(64), P(0)) == -1
    assert lib.medusa_buffers_restore(P(16), P(8), P(8), U32(1), P(0), P(0), U32(3), P(64), P(0)) == -1


def test_no_cpu_fallback_without_gpu(lib):
    """On a host without a usable GPU, valid calls fail with MEDUSA_ERR_CUDA."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    assert lib.medusa_kernel_table_set(ctypes.c_void_p(0), ctypes.c_uint32(0), ctypes.c_void_p(0)) == -5
    P, U32 = ctypes.c_void_p, ctypes.c_uint32
    assert lib.medusa_buffers_restore(P(16), P(8), P(8), U32(0), P(0), P(0), U32(0), P(64), P(0)) == -5
