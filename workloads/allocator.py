"""PyTorch-caching-allocator-like simulator used ONLY to synthesise inputs.

This module is part of the seeded input generator (``workloads/``).  It holds
none of the method's arithmetic: it never classifies a word against a trace.
It only plays the role of the allocator whose (de)allocation sequence Medusa
intercepts and keeps the bookkeeping a real
allocator has (which blocks are handed out right now).

Model ([ext] PyTorch c10 CUDACachingAllocator, simplified):
  * requests are rounded up to 512 B;
  * small pool: requests <= 1 MiB, carved from 2 MiB segments; a block is split
    when the remainder is >= 512 B;
  * large pool: requests > 1 MiB, segments of 20 MiB (request < 10 MiB) or the
    request rounded up to 2 MiB; a block is split when the remainder > 1 MiB;
  * best fit = the smallest free block whose size >= request (ties: lowest
    address); freed blocks coalesce with free neighbours of the same segment;
  * segments are never returned (no empty_cache), so addresses get reused
    across layers, forwards and graphs exactly as in Fig. 6;
  * pools are independent (the default pool and the CUDA-graph private pool).
Segments are placed at increasing, 2 MiB aligned virtual addresses inside the
model's VA region with a 2-6 MiB hole after each one (holes are never
allocated; they host the "gap" adversarial words).
"""
from __future__ import annotations

from sortedcontainers import SortedDict, SortedList

KB = 1024
MiB = 1024 * 1024
ROUND = 512
SMALL_MAX = 1 * MiB
SMALL_SEG = 2 * MiB
LARGE_SEG = 20 * MiB
MIN_LARGE_ALLOC = 10 * MiB
ROUND_LARGE = 2 * MiB


def _round_up(x: int, m: int) -> int:
    return (x + m - 1) // m * m


class _Block:
    __slots__ = ("addr", "size", "seg", "prev", "next", "allocated", "small", "pool")

    def __init__(self, addr, size, seg, small, pool):
        self.addr = addr
        self.size = size
        self.seg = seg
        self.prev = None
        self.next = None
        self.allocated = False
        self.small = small
        self.pool = pool


class Segment:
    __slots__ = ("base", "size", "pool", "small", "index")

    def __init__(self, base, size, pool, small, index):
        self.base = base
        self.size = size
        self.pool = pool
        self.small = small
        self.index = index


class CachingAllocator:
    """Two-pool caching allocator over one VA region."""

    def __init__(self, va_base: int, rng):
        self.next_va = _round_up(va_base, ROUND_LARGE)
        self.va_base = va_base
        self.rng = rng
        self.segments: list[Segment] = []
        self._free = {}  # (pool, small) -> SortedList[(size, addr)]
        self._blocks = {}  # addr -> _Block (every block, free or not)
        self.gaps: list[tuple[int, int]] = []  # never-allocated VA holes

    # -- internals ---------------------------------------------------------
    def _fl(self, pool, small):
        key = (pool, small)
        fl = self._free.get(key)
        if fl is None:
            fl = SortedList()
            self._free[key] = fl
        return fl

    def _new_segment(self, size: int, pool: str, small: bool) -> _Block:
        if small:
            seg_size = SMALL_SEG
        elif size < MIN_LARGE_ALLOC:
            seg_size = LARGE_SEG
        else:
            seg_size = _round_up(size, ROUND_LARGE)
        base = self.next_va
        seg = Segment(base, seg_size, pool, small, len(self.segments))
        self.segments.append(seg)
        hole = ROUND_LARGE * int(self.rng.integers(1, 4))
        self.gaps.append((base + seg_size, base + seg_size + hole))
        self.next_va = base + seg_size + hole
        blk = _Block(base, seg_size, seg, small, pool)
        self._blocks[base] = blk
        return blk

    # -- public API --------------------------------------------------------
    def malloc(self, nbytes: int, pool: str = "default") -> tuple[int, int, Segment]:
        """Return (address, recorded size, segment). Recorded size = request
        rounded to 512 B (the tensor's extent), not the possibly larger block."""
        size = _round_up(max(int(nbytes), 1), ROUND)
        small = size <= SMALL_MAX
        fl = self._fl(pool, small)
        i = fl.bisect_left((size, -1))
        if i < len(fl):
            bsize, baddr = fl[i]
            del fl[i]
            blk = self._blocks[baddr]
        else:
            blk = self._new_segment(size, pool, small)
        remaining = blk.size - size
        if (small and remaining >= ROUND) or ((not small) and remaining > SMALL_MAX):
            rest = _Block(blk.addr + size, remaining, blk.seg, small, pool)
            rest.prev = blk
            rest.next = blk.next
            if blk.next is not None:
                blk.next.prev = rest
            blk.next = rest
            blk.size = size
            self._blocks[rest.addr] = rest
            fl.add((rest.size, rest.addr))
        blk.allocated = True
        return blk.addr, size, blk.seg

    def free(self, addr: int) -> None:
        blk = self._blocks[addr]
        assert blk.allocated, "double free in generator"
        blk.allocated = False
        fl = self._fl(blk.pool, blk.small)
        prev = blk.prev
        if prev is not None and not prev.allocated:
            fl.remove((prev.size, prev.addr))
            prev.size += blk.size
            prev.next = blk.next
            if blk.next is not None:
                blk.next.prev = prev
            del self._blocks[blk.addr]
            blk = prev
        nxt = blk.next
        if nxt is not None and not nxt.allocated:
            fl.remove((nxt.size, nxt.addr))
            blk.size += nxt.size
            blk.next = nxt.next
            if nxt.next is not None:
                nxt.next.prev = blk
            del self._blocks[nxt.addr]
        fl.add((blk.size, blk.addr))


class LiveSet:
    """Bookkeeping of the allocations handed out right now, as the trace
    records them (base, recorded size, allocation ordinal).  Used by the
    generator to place adversarial words whose category it must know."""

    def __init__(self):
        self._by_base = SortedDict()  # base -> (size, alloc_id)
        self._ids = []  # dense list of live ids for O(1) random choice
        self._pos = {}

    def add(self, base, size, aid):
        self._by_base[base] = (size, aid)
        self._pos[aid] = len(self._ids)
        self._ids.append(aid)

    def remove(self, base, aid):
        del self._by_base[base]
        p = self._pos.pop(aid)
        last = self._ids.pop()
        if last != aid:
            self._ids[p] = last
            self._pos[last] = p

    def covering(self, addr):
        """alloc id whose recorded [base, base+size) holds addr, else -1."""
        i = self._by_base.bisect_right(addr) - 1
        if i < 0:
            return -1
        base = self._by_base.keys()[i]
        size, aid = self._by_base[base]
        return aid if addr - base < size else -1

    def starting_at(self, addr):
        v = self._by_base.get(addr)
        return -1 if v is None else v[1]

    def random_id(self, rng):
        return self._ids[int(rng.integers(0, len(self._ids)))] if self._ids else -1

    def __len__(self):
        return len(self._ids)
