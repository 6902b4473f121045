"""ORACLE -- test infrastructure only (see oracle.cpp header).

Loads liboracle.so (plain C++, built by __graft_entry__.build()) with ctypes
and exposes numpy-in / numpy-out wrappers.  Only tests/, smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package.  The CUDA path
never imports it and it never imports the CUDA path.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
OK, ERR_INVALID_ARG, ERR_TRACE = 0, -1, -2
CHUNK_WORDS = 2048
_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(LIB_PATH)
        P, U64, U32, I = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        lib.oracle_check.argtypes = [U64, P, U32, P, P, U32]
        lib.oracle_check.restype = I
        lib.oracle_materialize.argtypes = [P, U64, P, U32, P, P, U32, P, P, P, P]
        lib.oracle_materialize.restype = I
        lib.oracle_pack_slots.argtypes = [P, P, P, U64, P, P, P]
        lib.oracle_pack_slots.restype = None
        lib.oracle_restore.argtypes = [P, P, U64, P, P, P, U64, P, P, P, U32, P, P, U32, P, U32, P]
        lib.oracle_restore.restype = None
        lib.oracle_restore_packed.argtypes = [P, P, U64, P, P, P, U64, P, P, P, U32, P, P, U32, P, U32, P]
        lib.oracle_restore_packed.restype = None
        _lib = lib
    return _lib


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None and a.size else ctypes.c_void_p(0)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def check(words_n, node_off, node_t, allocs) -> int:
    lib = _load()
    node_off = _c(node_off, np.uint64)
    node_t = _c(node_t, np.uint32)
    allocs = np.ascontiguousarray(allocs)
    assert allocs.dtype.itemsize == 24
    return lib.oracle_check(words_n, _p(node_off), node_t.size, _p(node_t), _p(allocs), allocs.size)


def materialize(words, node_off, node_t, allocs):
    """-> dict(status, is_slot[u8 n_words], id[u32], off[u64], n_slots, slot_g/slot_id/slot_off)."""
    lib = _load()
    words = _c(words, np.uint64)
    node_off = _c(node_off, np.uint64)
    node_t = _c(node_t, np.uint32)
    allocs = np.ascontiguousarray(allocs)
    n = words.size
    is_slot = np.zeros(max(n, 1), np.uint8)
    sid = np.zeros(max(n, 1), np.uint32)
    soff = np.zeros(max(n, 1), np.uint64)
    ns = ctypes.c_uint64(0)
    st = lib.oracle_materialize(_p(words), n, _p(node_off), node_t.size, _p(node_t), _p(allocs), allocs.size,
                                _p(is_slot), _p(sid), _p(soff), ctypes.byref(ns))
    is_slot, sid, soff = is_slot[:n], sid[:n], soff[:n]
    g = np.flatnonzero(is_slot).astype(np.uint64)
    return dict(status=st, n_slots=int(ns.value), is_slot=is_slot, id=sid, off=soff,
                slot_g=g, slot_id=sid[g.astype(np.int64)], slot_off=soff[g.astype(np.int64)])


def pack(m, n_words):
    """Slot list -> ABI layout (mask u32, chunk_base u32, records u64)."""
    lib = _load()
    n_mask = (n_words + 31) // 32
    n_chunks = (n_words + CHUNK_WORDS - 1) // CHUNK_WORDS
    mask = np.zeros(max(n_mask, 1), np.uint32)
    cb = np.zeros(n_chunks + 1, np.uint32)
    rec = np.zeros(max(m["n_slots"], 1), np.uint64)
    lib.oracle_pack_slots(_p(m["is_slot"]), _p(m["id"]), _p(m["off"]), n_words, _p(mask), _p(cb), _p(rec))
    return mask[:n_mask], cb, rec[: m["n_slots"]]


REPORT_FIELDS = ("n_bad_slot", "first_bad_word", "n_bad_id", "n_bad_range", "n_stale",
                 "n_bad_func", "first_bad_node", "n_bad_chunk")


def restore(src, slot_g, slot_id, slot_off, old_base, new_base, new_size, func_id=None, table=None):
    """-> (dst u64[n_words], func_out u64[N] or None, report u64[8])."""
    lib = _load()
    src = _c(src, np.uint64)
    dst = np.zeros_like(src)
    slot_g, slot_id, slot_off = _c(slot_g, np.uint64), _c(slot_id, np.uint32), _c(slot_off, np.uint64)
    old_base, new_base, new_size = _c(old_base, np.uint64), _c(new_base, np.uint64), _c(new_size, np.uint64)
    rep = np.zeros(8, np.uint64)
    fout = None
    if func_id is not None:
        func_id = _c(func_id, np.uint32)
        table = _c(table, np.uint64)
        fout = np.zeros(func_id.size, np.uint64)
    lib.oracle_restore(_p(src), _p(dst), src.size, _p(slot_g), _p(slot_id), _p(slot_off), slot_g.size,
                       _p(old_base), _p(new_base), _p(new_size), new_base.size,
                       _p(func_id) if func_id is not None else ctypes.c_void_p(0),
                       _p(fout) if fout is not None else ctypes.c_void_p(0),
                       func_id.size if func_id is not None else 0,
                       _p(table) if table is not None else ctypes.c_void_p(0),
                       table.size if table is not None else 0, _p(rep))
    return dst, fout, rep


def restore_packed(src, mask, chunk_base, records, n_slots, old_base, new_base, new_size, func_id=None,
                   table=None):
    """oracle_restore_packed (DESIGN.md R-TABLE) -> (dst u64[n_words], func_out or None, report u64[8])."""
    lib = _load()
    src = _c(src, np.uint64)
    dst = np.zeros_like(src)
    mask, chunk_base, records = _c(mask, np.uint32), _c(chunk_base, np.uint32), _c(records, np.uint64)
    assert chunk_base.size == (src.size + CHUNK_WORDS - 1) // CHUNK_WORDS + 1 and mask.size >= (src.size + 31) // 32
    assert records.size >= min(int(n_slots), int(chunk_base.max(initial=0)))
    old_base, new_base, new_size = _c(old_base, np.uint64), _c(new_base, np.uint64), _c(new_size, np.uint64)
    rep = np.zeros(8, np.uint64)
    fout = None
    if func_id is not None:
        func_id = _c(func_id, np.uint32)
        table = _c(table, np.uint64)
        fout = np.zeros(func_id.size, np.uint64)
    lib.oracle_restore_packed(_p(src), _p(dst), src.size, _p(mask), _p(chunk_base), _p(records), int(n_slots),
                              _p(old_base), _p(new_base), _p(new_size), new_base.size,
                              _p(func_id) if func_id is not None else ctypes.c_void_p(0),
                              _p(fout) if fout is not None else ctypes.c_void_p(0),
                              func_id.size if func_id is not None else 0,
                              _p(table) if table is not None else ctypes.c_void_p(0),
                              table.size if table is not None else 0, _p(rep))
    return dst, fout, rep
