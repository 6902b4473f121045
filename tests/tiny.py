"""Tiny adversarial traces for brute-force comparisons (P3) and edge cases.

A seeded random process of allocation / free / launch events over a small
address window, with heavy address reuse (Fig. 6), adjacency (one-past-end),
dangling words, zero-size allocations and equal event positions across kinds.
Well-formed unless `overlap_p` > 0, in which case an allocation may be placed on
top of a live one (a malformed trace the oracle must reject).
"""
from __future__ import annotations

import numpy as np

from workloads import ALLOC_DTYPE, T_NEVER

BASE0 = 0x7F00_0000_0000


def tiny_trace(seed, n_steps=120, overlap_p=0.0, max_words=6, max_allocs=60):
    rng = np.random.default_rng(seed)
    allocs = []  # [base, size, ta, tf]
    live = []
    nodes_t, nodes_w = [], []
    t = 1
    last_alloc_t = 0
    last_launch_t = 0
    for _ in range(n_steps):
        r = rng.random()
        t += int(rng.choice([0, 1, 1, 2]))
        if r < 0.35 and len(allocs) < max_allocs:
            tt = max(t, last_alloc_t + 1)
            size = int(rng.choice([0, 16, 64, 64, 128, 192, 256]))
            for _try in range(8):
                base = BASE0 + 64 * int(rng.integers(0, 24)) + 16 * int(rng.integers(0, 2))
                clash = any(size > 0 and a[1] > 0 and base < a[0] + a[1] and a[0] < base + size
                            for a in (allocs[i] for i in live))
                if not clash or rng.random() < overlap_p:
                    break
            else:
                continue
            t = tt
            last_alloc_t = tt
            allocs.append([base, size, tt, T_NEVER])
            live.append(len(allocs) - 1)
        elif r < 0.6 and live:
            i = live.pop(int(rng.integers(0, len(live))))
            tt = max(t, allocs[i][2] + 1)
            t = tt
            allocs[i][3] = tt
        else:
            tt = max(t, last_launch_t + 1)
            t = tt
            last_launch_t = tt
            ws = []
            for _w in range(int(rng.integers(0, max_words + 1))):
                k = rng.random()
                if k < 0.4 and allocs:
                    a = allocs[int(rng.integers(0, len(allocs)))]
                    ws.append(a[0] + int(rng.integers(0, max(a[1], 1) + 1)))  # interior / one past end
                elif k < 0.55:
                    ws.append(BASE0 + int(rng.integers(0, 24 * 64 + 256)))
                elif k < 0.7:
                    ws.append(int(rng.integers(0, 1 << 32)))
                elif k < 0.8:
                    ws.append(0)
                else:
                    ws.append(int(rng.integers(0, 1 << 63)) * 2 + int(rng.integers(0, 2)))
            nodes_t.append(tt)
            nodes_w.append(ws)
    arr = np.zeros(len(allocs), ALLOC_DTYPE)
    for i, (b, s, ta, tf) in enumerate(allocs):
        arr[i] = (b, s, ta, tf)
    words = np.array([w for ws in nodes_w for w in ws], dtype=np.uint64)
    off = np.zeros(len(nodes_w) + 1, np.uint64)
    off[1:] = np.cumsum([len(ws) for ws in nodes_w])
    return words, off, np.array(nodes_t, np.uint32), arr


def as_tuples(allocs):
    return [(int(a["base"]), int(a["size"]), int(a["t_alloc"]), int(a["t_free"])) for a in allocs]
