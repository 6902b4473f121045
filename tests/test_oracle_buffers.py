"""Pins of the buffer-contents oracle (oracle/buffers.py, §4.3).

B1 hand-built trace with every class (tests/golden/buffers.json)
B2 generator ground truth: the PERM buffers are exactly the two 4-byte buffers
   of every permanent-buffer kernel; weights / KV / static inputs are
   PARAM; capture temporaries TEMP; profiling and warm-up
   buffers are never referenced
B3 identity: saving and restoring onto the same addresses changes nothing
B4 round trip: after restore, every PERM buffer's new range holds the bytes
   its old range held; no other byte of the new memory changes
B5 validation faults land in the count with the least segment index
B6 malformed capture intervals are rejected
"""
import json
import os

import numpy as np
import pytest

import oracle
from oracle import buffers as ob
from workloads import ALLOC_DTYPE, T_NEVER
from workloads.graphset import AK_CAPTURE, AK_KV, AK_PERM, AK_PROFILE, AK_STATIC, AK_WARMUP, AK_WEIGHT

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
NAMES = {"UNUSED": ob.UNUSED, "PARAM": ob.PARAM, "TEMP": ob.TEMP, "PERM": ob.PERM}


def _fixture():
    fx = json.load(open(os.path.join(GOLDEN, "buffers.json")))
    a = np.zeros(len(fx["allocs"]), ALLOC_DTYPE)
    for i, r in enumerate(fx["allocs"]):
        a[i] = (r["base"], r["size"], r["t_alloc"], r["t_free"])
    return fx, a


def test_b1_hand_built_trace():
    fx, a = _fixture()
    cls = ob.classify(a, fx["captures"], fx["slot_ids"])
    assert [int(c) for c in cls] == [NAMES[c] for c in fx["expected_class"]]
    perm, off = ob.plan(a, cls)
    assert perm.tolist() == fx["expected_perm"] and off.tolist() == fx["expected_off"]


def _slots(gs):
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    assert m["status"] == 0
    return m["slot_id"]


@pytest.mark.parametrize("name", ["toy", "llama2-7b"])
def test_b2_generator_ground_truth(graph_sets, name):
    gs = graph_sets(name)
    sid = _slots(gs)
    cls = ob.classify(gs.allocs, gs.capture_t, sid)
    ref = np.zeros(gs.n_alloc, bool)
    ref[sid] = True
    k = gs.alloc_kind
    # every permanent buffer is referenced, and is exactly what PERM finds
    assert ref[k == AK_PERM].all()
    assert np.array_equal(cls == ob.PERM, k == AK_PERM)
    # two permanent buffers per permanent-buffer kernel, each "only 4 bytes":
    # the trace records the 4-byte request at the allocator's 512-B rounding
    assert int((cls == ob.PERM).sum()) == 2 * int(gs.node_perm.sum())
    assert (gs.allocs["size"][cls == ob.PERM] == 512).all()
    # model parameters and everything else prepared before capture
    pre = np.isin(k, [AK_WEIGHT, AK_KV, AK_STATIC])
    assert (cls[pre & ref] == ob.PARAM).all() and (cls[pre & ~ref] == ob.UNUSED).all()
    # capture temporaries are deallocated after capturing
    assert (cls[(k == AK_CAPTURE) & ref] == ob.TEMP).all()
    # profiling / warm-up buffers are dead at every captured launch
    assert (cls[np.isin(k, [AK_PROFILE, AK_WARMUP])] == ob.UNUSED).all()
    perm, off = ob.plan(gs.allocs, cls)
    assert int(off[-1]) == 512 * perm.size


def _arena_case(rng, n_perm=6):
    """Allocations whose bases are real offsets into an arena (old) and a
    second arena (new), PERM ones among them."""
    sizes = rng.choice([8, 24, 512, 1000, 4096], size=3 * n_perm)
    a = np.zeros(sizes.size, ALLOC_DTYPE)
    old_base, new_base = 1 << 20, 1 << 30
    po, pn = 0, 0
    order = rng.permutation(sizes.size)
    newpos = np.zeros(sizes.size, np.int64)
    for i in order:  # the replay places allocations in another order
        newpos[i] = pn
        pn += int(sizes[i]) + 8 * int(rng.integers(0, 4))
    for i, s in enumerate(sizes):
        a[i] = (old_base + po, s, 2 * i + 1, T_NEVER)
        po += int(s) + 8 * int(rng.integers(0, 4))
    cls = np.zeros(sizes.size, np.uint8)
    cls[rng.choice(sizes.size, size=n_perm, replace=False)] = ob.PERM
    nb = (new_base + newpos).astype(np.uint64)
    old = ob.Arena(old_base, data=rng.integers(0, 256, size=po, dtype=np.uint8))
    new = ob.Arena(new_base, data=np.full(pn, 0xA5, np.uint8))
    return a, cls, old, new, nb


def test_b3_identity():
    rng = np.random.default_rng(5)
    a, cls, old, _, _ = _arena_case(rng)
    perm, off = ob.plan(a, cls)
    blob = ob.save(old, perm, off, a["base"])
    before = old.data.copy()
    assert ob.restore(old, blob, perm, off, a["base"], a["size"]) == (0, (1 << 64) - 1)
    assert np.array_equal(old.data, before)


def test_b4_round_trip():
    rng = np.random.default_rng(6)
    a, cls, old, new, nb = _arena_case(rng)
    perm, off = ob.plan(a, cls)
    blob = ob.save(old, perm, off, a["base"])
    assert blob.size == int(a["size"][cls == ob.PERM].sum())
    poison = new.data.copy()
    assert ob.restore(new, blob, perm, off, nb, a["size"])[0] == 0
    touched = np.zeros(new.data.size, bool)
    for i in perm:
        s = int(a["size"][i])
        assert np.array_equal(new.read(int(nb[i]), s), old.read(int(a["base"][i]), s))
        touched[int(nb[i]) - new.base:int(nb[i]) - new.base + s] = True
    assert np.array_equal(new.data[~touched], poison[~touched])


def test_b5_faults():
    rng = np.random.default_rng(7)
    a, cls, old, new, nb = _arena_case(rng)
    perm, off = ob.plan(a, cls)
    blob = ob.save(old, perm, off, a["base"])
    size = a["size"].copy()
    size[perm[3]] -= 1                      # the replayed allocation is smaller
    n_bad, first = ob.restore(new, blob, perm, off, nb, size)
    assert (n_bad, first) == (1, 3)
    assert new.read(int(nb[perm[3]]), 4).tolist() == [0xA5] * 4   # not restored
    short = nb[: int(perm[-1])]              # the replay made fewer allocations
    n_bad, first = ob.restore(new, blob, perm, off, short, size)
    assert n_bad == 2 and first == 3


def test_b6_capture_checks():
    assert ob.check_captures([[1, 5], [5, 9]]) == ob.OK
    assert ob.check_captures([[1, 5], [4, 9]]) == ob.ERR_INVALID_ARG
    assert ob.check_captures([[6, 5]]) == ob.ERR_INVALID_ARG
    assert ob.check_captures([[6, 9], [1, 2]]) == ob.ERR_INVALID_ARG
    assert ob.check_captures(np.zeros((0, 2))) == ob.OK
