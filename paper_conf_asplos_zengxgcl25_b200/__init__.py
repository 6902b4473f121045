"""Thin Python binding of libmedusa.so (include/medusa.h).

Argument marshalling only: torch tensors supply device memory and streams;
every step of the path runs in the library's sm_100a kernels.  There is no CPU
fallback -- if libmedusa.so is missing or a call fails, an exception is raised.

Names follow the C ABI: materialize, kernel_table_set, restore.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
# MEDUSA_LIB: a diagnostic build variant of the same library (tools/, A/B runs)
LIB_PATH = os.environ.get("MEDUSA_LIB") or os.path.join(_HERE, "libmedusa.so")

OK, ERR_INVALID_ARG, ERR_TRACE, ERR_CAPACITY, ERR_NO_TABLE, ERR_CUDA, ERR_RETRY = 0, -1, -2, -3, -4, -5, -6
N_SLOTS_FROM_TABLE = (1 << 64) - 1
CHUNK_WORDS = 2048
OFF_BITS = 40
T_END = 0xFFFFFFFF
REPORT_FIELDS = ("n_bad_slot", "first_bad_word", "n_bad_id", "n_bad_range", "n_stale",
                 "n_bad_func", "first_bad_node", "n_bad_chunk")


class MedusaError(RuntimeError):
    def __init__(self, status, what, n_slots=None):
        self.status = status
        self.n_slots = n_slots
        extra = ""
        if status == ERR_CUDA:
            extra = f" (cudaError {lib().medusa_last_cuda_error()})"
        super().__init__(f"{what}: {lib().medusa_status_string(status).decode()}{extra}")


class _Slots(ctypes.Structure):
    _fields_ = [("d_mask", ctypes.c_void_p), ("d_chunk_base", ctypes.c_void_p), ("d_slot", ctypes.c_void_p),
                ("capacity", ctypes.c_uint64)]


_lib = None


def lib():
    """The loaded libmedusa.so (raises if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing; run __graft_entry__.build() -- there is no fallback")
        L = ctypes.CDLL(LIB_PATH)
        P, U64, U32, I = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        L.medusa_materialize.argtypes = [P, U64, P, U32, P, P, U32, ctypes.POINTER(_Slots),
                                         ctypes.POINTER(U64), P]
        L.medusa_materialize.restype = I
        L.medusa_materialize_async.argtypes = [P, U64, P, U32, P, P, U32, ctypes.POINTER(_Slots), P, P]
        L.medusa_materialize_async.restype = I
        L.medusa_kernel_table_set.argtypes = [P, U32, P]
        L.medusa_kernel_table_set.restype = I
        L.medusa_restore.argtypes = [P, P, U64, ctypes.POINTER(_Slots), U64, P, P, P, U32, P, P, U32, P, P]
        L.medusa_restore.restype = I
        L.medusa_buffers_plan.argtypes = [P, U32, P, U32, P, U64, P, P, P, U32, ctypes.POINTER(U32),
                                          ctypes.POINTER(U64), P]
        L.medusa_buffers_plan.restype = I
        L.medusa_buffers_save.argtypes = [P, P, U32, P, U32, P, P, P]
        L.medusa_buffers_save.restype = I
        L.medusa_buffers_restore.argtypes = [P, P, P, U32, P, P, U32, P, P]
        L.medusa_buffers_restore.restype = I
        L.medusa_last_cuda_error.argtypes = []
        L.medusa_last_cuda_error.restype = I
        L.medusa_status_string.argtypes = [I]
        L.medusa_status_string.restype = ctypes.c_char_p
        L.medusa_timing_enable.argtypes = [I]
        L.medusa_timing_enable.restype = None
        L.medusa_timing_read.argtypes = [ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(ctypes.c_float), I]
        L.medusa_timing_read.restype = I
        L.medusa_scratch_bytes.argtypes = []
        L.medusa_scratch_bytes.restype = U64
        L.medusa_scratch_release.argtypes = []
        L.medusa_scratch_release.restype = I
        _lib = L
    return _lib


lib()  # fail loudly at import if the native library is absent


def _ptr(t):
    if t is None:
        return ctypes.c_void_p(0)
    return ctypes.c_void_p(t.data_ptr() if t.numel() else 0)


def _stream(stream):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


class Slots:
    """The materialized indirect-index-pointer table (device tensors)."""

    def __init__(self, mask, chunk_base, slot, n_slots):
        self.mask = mask  # int32[ceil(n_words/32)]
        self.chunk_base = chunk_base  # int32[ceil(n_words/2048)+1]
        self.slot = slot  # int64[capacity]
        self.n_slots = int(n_slots)

    @property
    def capacity(self):
        return int(self.slot.numel())

    def c_struct(self):
        return _Slots(self.mask.data_ptr() if self.mask.numel() else 0, self.chunk_base.data_ptr(),
                      self.slot.data_ptr() if self.slot.numel() else 0, self.capacity)


def alloc_slots(n_words, device, capacity=None):
    if capacity is None:
        capacity = n_words
    return Slots(torch.empty(max((n_words + 31) // 32, 0), dtype=torch.int32, device=device),
                 torch.empty((n_words + CHUNK_WORDS - 1) // CHUNK_WORDS + 1, dtype=torch.int32, device=device),
                 torch.empty(capacity, dtype=torch.int64, device=device), 0)


def materialize(words, node_off, node_t, allocs, stream=None, capacity=None, out=None):
    """medusa_materialize.  words int64[n_words], node_off int64[N+1], node_t int32[N],
    allocs int64[n_alloc, 3] (the 24-byte medusa_alloc records) -> Slots."""
    n_words = words.numel()
    slots = out if out is not None else alloc_slots(n_words, words.device, capacity)
    cs = slots.c_struct()
    n = ctypes.c_uint64(0)
    st = lib().medusa_materialize(_ptr(words), n_words, _ptr(node_off), node_t.numel(), _ptr(node_t),
                                  _ptr(allocs), allocs.shape[0] if allocs.dim() else 0, ctypes.byref(cs),
                                  ctypes.byref(n), _stream(stream))
    if st != OK:
        raise MedusaError(st, "medusa_materialize", int(n.value))
    slots.n_slots = int(n.value)
    return slots


def materialize_async(words, node_off, node_t, allocs, out, result, stream=None):
    """medusa_materialize_async: enqueue only.  `result` = int64[2] device tensor that
    receives {status (low 32 bits of [0]), n_slots ([1])}; `out` = a Slots sized for
    this image (its n_slots is not updated -- read `result` or restore with
    from_table=True)."""
    cs = out.c_struct()
    st = lib().medusa_materialize_async(_ptr(words), words.numel(), _ptr(node_off), node_t.numel(), _ptr(node_t),
                                        _ptr(allocs), allocs.shape[0] if allocs.dim() else 0, ctypes.byref(cs),
                                        _ptr(result), _stream(stream))
    if st != OK:
        raise MedusaError(st, "medusa_materialize_async")
    return out


def mat_result(result):
    """(status, n_slots) from a materialize_async result tensor (synchronizes)."""
    r = result.detach().cpu().numpy()
    return int(np.int32(r[0] & 0xFFFFFFFF)), int(r[1])


def kernel_table_set(table, stream=None):
    """medusa_kernel_table_set.  table: int64[K] device tensor of kernel addresses (0 = unresolved)."""
    st = lib().medusa_kernel_table_set(_ptr(table), table.numel(), _stream(stream))
    if st != OK:
        raise MedusaError(st, "medusa_kernel_table_set")


def restore(src, slots, old_base, new_base, new_size, func_id=None, dst=None, func_out=None, report=None,
            stream=None, from_table=False):
    """medusa_restore -> (dst int64[n_words], func_out int64[N] or None, report int64[8]).
    dst may be src (in place).  from_table: slot count taken from the table itself
    (MEDUSA_N_SLOTS_FROM_TABLE), e.g. after materialize_async."""
    dev = src.device
    if dst is None:
        dst = torch.empty_like(src)
    if func_id is not None and func_out is None:
        func_out = torch.empty(func_id.numel(), dtype=torch.int64, device=dev)
    if report is None:
        report = torch.empty(8, dtype=torch.int64, device=dev)
    cs = slots.c_struct()
    n_slots = N_SLOTS_FROM_TABLE if from_table else slots.n_slots
    st = lib().medusa_restore(_ptr(src), _ptr(dst), src.numel(), ctypes.byref(cs), n_slots, _ptr(old_base),
                              _ptr(new_base), _ptr(new_size), new_base.numel(), _ptr(func_id), _ptr(func_out),
                              func_id.numel() if func_id is not None else 0, _ptr(report), _stream(stream))
    if st != OK:
        raise MedusaError(st, "medusa_restore")
    return dst, func_out, report


BUF_UNUSED, BUF_PARAM, BUF_TEMP, BUF_PERM = 0, 1, 2, 3


class BufferPlan:
    """Output of medusa_buffers_plan (device tensors): class per allocation, the
    permanent allocations and the blob layout."""

    def __init__(self, cls, perm, perm_off, n_perm, blob_bytes):
        self.cls = cls  # uint8[n_alloc]
        self.perm = perm  # int32[n_perm] allocation indices
        self.perm_off = perm_off  # int64[n_perm + 1] blob offsets
        self.n_perm = int(n_perm)
        self.blob_bytes = int(blob_bytes)


def buffers_plan(allocs, capture_t, slot, n_slots, stream=None, capacity=None):
    """medusa_buffers_plan.  allocs int64[n_alloc, 3] (medusa_alloc records), capture_t
    int32[n_capture, 2] (begin, end) event positions, slot int64[>= n_slots] (the
    materialized records, e.g. Slots.slot) -> BufferPlan.  capacity defaults to
    n_alloc (always enough)."""
    dev = allocs.device
    n_alloc = allocs.shape[0] if allocs.dim() else 0
    cap = n_alloc if capacity is None else int(capacity)
    cls = torch.empty(max(n_alloc, 1), dtype=torch.uint8, device=dev)
    perm = torch.empty(max(cap, 1), dtype=torch.int32, device=dev)
    perm_off = torch.empty(cap + 1, dtype=torch.int64, device=dev)
    n_perm, nbytes = ctypes.c_uint32(0), ctypes.c_uint64(0)
    st = lib().medusa_buffers_plan(_ptr(allocs), n_alloc, _ptr(capture_t), capture_t.numel() // 2,
                                   _ptr(slot), int(n_slots), _ptr(cls), _ptr(perm), _ptr(perm_off), cap,
                                   ctypes.byref(n_perm), ctypes.byref(nbytes), _stream(stream))
    if st != OK:
        e = MedusaError(st, "medusa_buffers_plan")
        e.n_perm, e.blob_bytes = int(n_perm.value), int(nbytes.value)
        raise e
    n = int(n_perm.value)
    return BufferPlan(cls[:n_alloc], perm[:n], perm_off[:n + 1], n, nbytes.value)


def buffers_save(plan, base, blob=None, report=None, stream=None):
    """medusa_buffers_save: blob uint8[plan.blob_bytes] <- the PERM buffers' bytes at
    base[i] (int64[n_alloc] device addresses) -> (blob, report int64[2])."""
    dev = base.device
    if blob is None:
        blob = torch.empty(max(plan.blob_bytes, 16), dtype=torch.uint8, device=dev)
    if report is None:
        report = torch.empty(2, dtype=torch.int64, device=dev)
    st = lib().medusa_buffers_save(_ptr(plan.perm), _ptr(plan.perm_off), plan.n_perm, _ptr(base), base.numel(),
                                   _ptr(blob), _ptr(report), _stream(stream))
    if st != OK:
        raise MedusaError(st, "medusa_buffers_save")
    return blob, report


def buffers_restore(plan, blob, new_base, new_size, report=None, stream=None):
    """medusa_buffers_restore: copy each saved segment to its replayed allocation
    -> report int64[2] (n_bad, first_bad)."""
    if report is None:
        report = torch.empty(2, dtype=torch.int64, device=blob.device)
    st = lib().medusa_buffers_restore(_ptr(blob), _ptr(plan.perm), _ptr(plan.perm_off), plan.n_perm,
                                      _ptr(new_base), _ptr(new_size), new_base.numel(), _ptr(report),
                                      _stream(stream))
    if st != OK:
        raise MedusaError(st, "medusa_buffers_restore")
    return report


def scratch_bytes():
    """medusa_scratch_bytes: live materialize scratch of the current device."""
    return int(lib().medusa_scratch_bytes())


def scratch_release():
    """medusa_scratch_release: free the current device's scratch and retired buffers
    (synchronizes; invalidates CUDA graphs that captured a materialize)."""
    st = lib().medusa_scratch_release()
    if st != OK:
        raise MedusaError(st, "medusa_scratch_release")


def timing_enable(on=True):
    lib().medusa_timing_enable(1 if on else 0)


def timing_read(max_n=4096):
    names = (ctypes.c_char_p * max_n)()
    ms = (ctypes.c_float * max_n)()
    n = lib().medusa_timing_read(names, ms, max_n)
    return [(names[i].decode(), float(ms[i])) for i in range(n)]


# ---- marshalling helpers (numpy <-> torch) ---------------------------------
def _t(a, dtype, device):
    return torch.from_numpy(np.ascontiguousarray(a)).to(device=device, dtype=dtype) if a.size else \
        torch.empty(0, dtype=dtype, device=device)


def host_arrays(gs):
    """numpy views of a graph set in the ABI dtypes (int64/int32 bit patterns)."""
    allocs = np.ascontiguousarray(gs.allocs)
    return dict(
        words=np.ascontiguousarray(gs.words).view(np.int64),
        node_off=np.ascontiguousarray(gs.node_word_off).view(np.int64),
        node_t=np.ascontiguousarray(gs.node_t).view(np.int32),
        allocs=allocs.view(np.int64).reshape(-1, 3) if allocs.size else np.zeros((0, 3), np.int64),
        old_base=np.ascontiguousarray(allocs["base"]).view(np.int64),
        new_base=np.ascontiguousarray(gs.new_base).view(np.int64),
        new_size=np.ascontiguousarray(gs.new_size).view(np.int64),
        func_id=np.ascontiguousarray(gs.func_id).view(np.int32),
        table=np.ascontiguousarray(gs.table).view(np.int64),
        capture_t=np.ascontiguousarray(gs.capture_t, dtype=np.uint32).view(np.int32).reshape(-1, 2),
    )


def upload(gs, device):
    """Copy a graph set's arrays to `device` (plumbing for tests / bench)."""
    h = host_arrays(gs)
    out = {}
    for k, v in h.items():
        out[k] = torch.from_numpy(v).to(device) if v.size else torch.empty(v.shape, dtype=torch.from_numpy(v).dtype,
                                                                            device=device)
    return out


def to_numpy_u64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def report_numpy(rep):
    return rep.detach().cpu().numpy().view(np.uint64)
