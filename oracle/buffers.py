"""ORACLE (test infrastructure only): copy-free buffer contents restoration.

PAPER.md §4.3, written out step by step in the paper's order.
Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this module.  It shares no code with the CUDA path
(paper_conf_asplos_zengxgcl25_b200/csrc/buffers.cu) and imports nothing from it.

  classify  -- which buffers' contents must be saved:
               "the buffer pointed by the CUDA graph nodes' parameters"
               = an allocation that at least one slot of the indirect index
               pointer table refers to;
               model-parameter buffers are "allocated before the CUDA graphs
               capturing" -> PARAM, skipped;
               temporary buffers are allocated during a capture and "deallocated
               after capturing" -> TEMP, skipped;
               the rest -- allocated during a capture, never deallocated -- are
               the permanent buffers "used across different launches of CUDA
               graphs" -> PERM, saved and restored.
               DESIGN.md readings R-B1..R-B4.
  plan      -- the PERM allocations in ordinal order and the exclusive prefix of
               their recorded sizes (the blob layout).
  save      -- offline: the contents of every PERM buffer, concatenated (P:220
               "dumping ... the buffer ... in the offline phase").
  restore   -- online: each saved segment copied to the replayed address of its
               allocation ("restoring them by reading and copying in the
               online phase"; P:176 the i-th allocation's new address), with
               the validation of DESIGN.md R-B4.

Memory is modelled by `Arena(base_address, bytes)`: device memory whose byte at
address a is bytes[a - base_address].

Pinned by tests/test_oracle_buffers.py: the generator's ground truth (every
PERM buffer is one of the two 4-byte buffers of a permanent-buffer kernel,
P:224; weights / KV / static inputs are PARAM; capture temporaries TEMP;
profiling and warm-up buffers never referenced), a hand-built trace with every
class, the identity and round-trip closed forms, and fault injection.
"""
from __future__ import annotations

import bisect

import numpy as np

T_END = 0xFFFFFFFF
UNUSED, PARAM, TEMP, PERM = 0, 1, 2, 3
OK, ERR_INVALID_ARG = 0, -1


class Arena:
    """A byte range of (device) memory starting at address `base`."""

    def __init__(self, base: int, nbytes: int | None = None, data: np.ndarray | None = None):
        self.base = int(base)
        self.data = np.zeros(int(nbytes), np.uint8) if data is None else np.array(data, np.uint8, copy=True)

    def read(self, addr: int, n: int) -> np.ndarray:
        o = int(addr) - self.base
        assert 0 <= o and o + n <= self.data.size, "address outside the arena"
        return self.data[o:o + n].copy()

    def write(self, addr: int, b: np.ndarray) -> None:
        o = int(addr) - self.base
        assert 0 <= o and o + b.size <= self.data.size, "address outside the arena"
        self.data[o:o + b.size] = b


def check_captures(capture_t) -> int:
    """Capture intervals (begin, end): begin < end, sorted and disjoint
    (graphs are captured one at a time)."""
    cap = [(int(b), int(e)) for b, e in np.asarray(capture_t, np.int64).reshape(-1, 2)]
    for k, (b, e) in enumerate(cap):
        if not b < e:
            return ERR_INVALID_ARG
        if k + 1 < len(cap) and not e <= cap[k + 1][0]:
            return ERR_INVALID_ARG
    return OK


def classify(allocs, capture_t, slot_id) -> np.ndarray:
    """-> u8[n_alloc] class of every allocation (UNUSED / PARAM / TEMP / PERM)."""
    n = int(allocs.size)
    cap = [(int(b), int(e)) for b, e in np.asarray(capture_t, np.int64).reshape(-1, 2)]
    begins = [b for b, _ in cap]
    # 1. the buffers pointed by the graph nodes' parameters
    referenced = np.zeros(n, bool)
    for i in np.asarray(slot_id, np.int64):
        if i < n:
            referenced[i] = True
    cls = np.zeros(n, np.uint8)
    for i in range(n):
        if not referenced[i]:
            continue
        t = int(allocs["t_alloc"][i])
        # 2. allocated during a capture?  The capture whose begin is the last one
        #    before t (intervals are sorted and disjoint) is the only candidate.
        k = bisect.bisect_left(begins, t) - 1
        during = k >= 0 and cap[k][0] < t < cap[k][1]
        if not during:
            cls[i] = PARAM          # "allocated before the CUDA graphs capturing"
        elif int(allocs["t_free"][i]) != T_END:
            cls[i] = TEMP           # "deallocated after capturing"
        else:
            cls[i] = PERM           # used across launches of the graph
    return cls


def plan(allocs, cls):
    """-> (perm u32[n_perm] ordinals in increasing order, off u64[n_perm+1]):
    segment k of the blob is [off[k], off[k+1]) and holds allocation perm[k]'s
    recorded size in bytes."""
    perm = np.array([i for i in range(cls.size) if cls[i] == PERM], np.uint32)
    off = np.zeros(perm.size + 1, np.uint64)
    for k, i in enumerate(perm):
        off[k + 1] = off[k] + np.uint64(allocs["size"][i])
    return perm, off


def save(mem: Arena, perm, off, base) -> np.ndarray:
    """Offline: blob = the bytes of every PERM buffer, at its address `base[i]`."""
    blob = np.zeros(int(off[-1]) if len(off) else 0, np.uint8)
    for k, i in enumerate(perm):
        n = int(off[k + 1] - off[k])
        blob[int(off[k]):int(off[k]) + n] = mem.read(int(base[i]), n)
    return blob


def restore(mem: Arena, blob, perm, off, new_base, new_size):
    """Online: copy segment k to new_base[perm[k]] unless perm[k] >= n_alloc of
    the replay or the segment is longer than the replayed allocation (R-B4).
    -> (n_bad, first_bad_k or 2^64-1); `mem` is modified in place."""
    n_alloc = len(new_base)
    n_bad, first = 0, (1 << 64) - 1
    for k, i in enumerate(perm):
        n = int(off[k + 1] - off[k])
        if int(i) >= n_alloc or n > int(new_size[i]):
            n_bad += 1
            first = min(first, k)
            continue
        mem.write(int(new_base[i]), np.asarray(blob[int(off[k]):int(off[k]) + n], np.uint8))
    return n_bad, first
