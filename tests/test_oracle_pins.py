"""Pins of the oracle against what the paper and mathematics fix (no GPU).

P1 Fig. 6 worked example      P7 round trip
P2 interior pointers / range rule        P8 generator ground truth
P3 literal backward scan == sweep        P9 Table 1 node totals
P4 identity relocation (closed form)             P10 9.0% / 69.2% statistics
P5 constant shift (closed form)                  P11 R1 vs R2 differ only on dead memory
P6 constants untouched                   P12 validation counters (R-Q8)
"""
import json
import os

import numpy as np
import pytest
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as st

import oracle
from oracle import brute
from tests.tiny import as_tuples, tiny_trace
from workloads import (ALLOC_DTYPE, ALL10, TABLE1_NODES, T_NEVER, TAG_CONST, TAG_DANGLING, TAG_FP, TAG_GAP,
                       TAG_OPE, TAG_PTR)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
U64 = (1 << 64) - 1


def _alloc_arr(rows):
    a = np.zeros(len(rows), ALLOC_DTYPE)
    for i, r in enumerate(rows):
        a[i] = tuple(int(x, 16) if isinstance(x, str) else int(x) for x in r)
    return a


def _slots_dict(m):
    return {int(g): (int(i), int(o)) for g, i, o in zip(m["slot_g"], m["slot_id"], m["slot_off"])}


# ---------------------------------------------------------------- P1
def test_p1_fig6_worked_example():
    fx = json.load(open(os.path.join(GOLDEN, "fig6.json")))
    allocs = _alloc_arr(fx["allocs"])
    words = np.array([int(w, 16) for n in fx["nodes"] for w in n["words"]], np.uint64)
    node_t = np.array([n["t"] for n in fx["nodes"]], np.uint32)
    off = np.array([0, 3, 6], np.uint64)
    m = oracle.materialize(words, off, node_t, allocs)
    assert m["status"] == 0
    exp = {int(k): tuple(v) for k, v in fx["expected_slots"].items()}
    assert _slots_dict(m) == exp
    assert brute.materialize(words, [0, 3, 6], node_t.tolist(), as_tuples(allocs), "R2") == exp
    # the naive address match is the paper's false positive and must differ on the second node
    naive = brute.materialize(words, [0, 3, 6], node_t.tolist(), as_tuples(allocs), "naive")
    assert naive == {int(k): tuple(v) for k, v in fx["naive_slots"].items()} and naive != exp
    new_base = np.array([int(x, 16) for x in fx["online_new_base"]], np.uint64)
    dst, _, rep = oracle.restore(words, m["slot_g"], m["slot_id"], m["slot_off"], allocs["base"], new_base,
                                 allocs["size"])
    assert [int(x) for x in dst] == [int(x, 16) for x in fx["expected_restored"]]
    assert rep[0] == 0
    # the naive table would restore A' for the t=6 node: data corruption
    ng = np.array(sorted(naive), np.uint64)
    nd, _, _ = oracle.restore(words, ng, [naive[g][0] for g in sorted(naive)], [naive[g][1] for g in sorted(naive)],
                              allocs["base"], new_base, allocs["size"])
    assert int(nd[3]) == int(new_base[1]) != int(dst[3])


# ---------------------------------------------------------------- P2
def test_p2_interior_pointers_and_range_ends():
    base, size = 0x7F00_0012_3400, 4096
    allocs = _alloc_arr([(base, size, 1, T_NEVER)])
    ks = list(range(0, 64)) + list(range(size - 64, size)) + [size // 2 + 1]
    vals = [base + k for k in ks] + [base + size, base - 1, base + size + 7, 0]
    words = np.array(vals, np.uint64)
    m = oracle.materialize(words, np.array([0, len(vals)], np.uint64), np.array([2], np.uint32), allocs)
    got = _slots_dict(m)
    for g, k in enumerate(ks):
        assert got[g] == (0, k)
    for g in range(len(ks), len(vals)):
        assert g not in got  # one-past-end, below base, above, null


def test_p2_zero_size_and_equal_positions():
    b = 0x7F00_0000_1000
    # allocation with size 0 never matches; launch at t == t_alloc or t == t_free sees nothing
    allocs = _alloc_arr([(b, 0, 1, T_NEVER), (b + 0x100, 64, 5, 9), (b + 0x200, 64, 10, T_NEVER)])
    words = np.array([b, b + 0x100, b + 0x100, b + 0x100, b + 0x200], np.uint64)
    off = np.array([0, 2, 3, 4, 5], np.uint64)
    node_t = np.array([5, 7, 9, 10], np.uint32)
    m = oracle.materialize(words, off, node_t, allocs)
    assert _slots_dict(m) == {2: (1, 0)}
    assert brute.materialize(words, off.tolist(), node_t.tolist(), as_tuples(allocs), "R2") == {2: (1, 0)}


# ---------------------------------------------------------------- P3
@settings(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(st.integers(0, 2**31 - 1), st.sampled_from([0.0, 0.0, 0.15]))
def test_p3_brute_equals_sweep(seed, overlap_p):
    words, off, node_t, allocs = tiny_trace(seed, overlap_p=overlap_p)
    ok = brute.check_trace_pairs(as_tuples(allocs))
    st_ = oracle.check(words.size, off, node_t, allocs)
    assert st_ == (oracle.OK if ok else oracle.ERR_TRACE)
    m = oracle.materialize(words, off, node_t, allocs)
    assert m["status"] == st_
    if ok:
        exp = brute.materialize(words, off.tolist(), node_t.tolist(), as_tuples(allocs), "R2")
        assert _slots_dict(m) == exp


def test_p3_malformed_and_invalid_inputs():
    b = 0x7F00_0000_0000
    ok_allocs = _alloc_arr([(b, 64, 1, 5), (b, 64, 5, 9)])  # free and re-alloc at the same position: fine
    off1 = np.array([0, 1], np.uint64)
    w1 = np.array([b], np.uint64)
    assert oracle.check(1, off1, np.array([6], np.uint32), ok_allocs) == oracle.OK
    bad = _alloc_arr([(b, 64, 1, 6), (b + 32, 64, 5, 9)])  # live at the same time, overlapping
    assert oracle.check(1, off1, np.array([7], np.uint32), bad) == oracle.ERR_TRACE
    assert not brute.check_trace_pairs(as_tuples(bad))
    assert oracle.check(1, off1, np.array([7], np.uint32), _alloc_arr([(b, 64, 3, 3)])) == oracle.ERR_TRACE
    assert oracle.check(1, off1, np.array([7], np.uint32), _alloc_arr([(b, 8, 4, 9), (b + 64, 8, 4, 9)])) == oracle.ERR_TRACE
    # invalid arguments
    assert oracle.check(1, off1, np.array([7], np.uint32), _alloc_arr([(b, (1 << 40) + 1, 1, 9)])) == oracle.ERR_INVALID_ARG
    assert oracle.check(1, off1, np.array([7], np.uint32), _alloc_arr([(U64 - 10, 64, 1, 9)])) == oracle.ERR_INVALID_ARG
    assert oracle.check(2, off1, np.array([7], np.uint32), ok_allocs) == oracle.ERR_INVALID_ARG
    assert oracle.check(2, np.array([0, 2, 1], np.uint64), np.array([7, 8], np.uint32), ok_allocs) == oracle.ERR_INVALID_ARG
    assert oracle.check(2, np.array([0, 1, 2], np.uint64), np.array([8, 8], np.uint32), ok_allocs) == oracle.ERR_INVALID_ARG
    assert oracle.check(2, np.array([1, 1, 2], np.uint64), np.array([7, 8], np.uint32), ok_allocs) == oracle.ERR_INVALID_ARG
    m = oracle.materialize(w1, off1, np.array([7], np.uint32), bad)
    assert m["status"] == oracle.ERR_TRACE and m["n_slots"] == 0


# ------------------------------------------------------------ P4 P5 P6 P7
@pytest.mark.parametrize("name", ["toy", "llama2-7b"])
def test_p4_p5_p6_p7_closed_forms(graph_sets, name):
    gs = graph_sets(name)
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    assert m["status"] == 0
    old = gs.allocs["base"]
    slot = m["is_slot"].astype(bool)
    # P4 identity
    dst, _, rep = oracle.restore(gs.words, m["slot_g"], m["slot_id"], m["slot_off"], old, old, gs.allocs["size"])
    assert np.array_equal(dst, gs.words) and rep[0] == 0
    # P5 constant shift by delta (mod 2^64)
    delta = np.uint64(0x1234_5600_0000)
    dst, _, rep = oracle.restore(gs.words, m["slot_g"], m["slot_id"], m["slot_off"], old, old + delta,
                                 gs.allocs["size"])
    assert np.array_equal(dst[slot], gs.words[slot] + delta) and np.array_equal(dst[~slot], gs.words[~slot])
    # P6 + P7: replayed addresses; every non-slot word bit-identical; round trip
    dst, _, rep = oracle.restore(gs.words, m["slot_g"], m["slot_id"], m["slot_off"], old, gs.new_base, gs.new_size)
    assert rep[0] == 0
    assert np.array_equal(dst[~slot], gs.words[~slot])
    assert np.array_equal(dst[slot], gs.new_base[m["id"][slot]] + m["off"][slot])
    new_allocs = gs.allocs.copy()
    new_allocs["base"] = gs.new_base
    m2 = oracle.materialize(dst, gs.node_word_off, gs.node_t, new_allocs)
    assert m2["status"] == 0
    for k in ("slot_g", "slot_id", "slot_off"):
        assert np.array_equal(m2[k], m[k])


# ---------------------------------------------------------------- P8
@pytest.mark.parametrize("name", ["toy", "qwen1.5-4b", "all10-inband"])
def test_p8_generator_ground_truth(graph_sets, name):
    gs = graph_sets(name)
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    slot = m["is_slot"].astype(bool)
    tags = gs.tags
    ptr = tags == TAG_PTR
    assert slot[ptr].all(), "recall on generated pointers must be 100%"
    assert np.array_equal(m["id"][ptr], gs.truth_id[ptr]) and np.array_equal(m["off"][ptr], gs.truth_off[ptr])
    fp = tags == TAG_FP
    assert slot[fp].all() and np.array_equal(m["id"][fp], gs.truth_id[fp])
    ope = tags == TAG_OPE
    adj = ope & (gs.truth_id >= 0)
    assert np.array_equal(slot[ope], adj[ope])
    assert np.array_equal(m["id"][adj], gs.truth_id[adj]) and (m["off"][adj] == 0).all()
    for tg in (TAG_CONST, TAG_GAP, TAG_DANGLING):
        assert not slot[tags == tg].any()
    extra = slot & ~ptr
    assert extra.sum() == fp.sum() + adj.sum()


# ---------------------------------------------------------------- P9 P10
def test_p9_table1_node_totals(graph_sets):
    gs = graph_sets("all10")
    for mi, name in enumerate(ALL10):
        assert int((gs.node_model == mi).sum()) == TABLE1_NODES[name]
    assert gs.n_nodes == 139364 == sum(TABLE1_NODES.values())
    for name in ("toy",):
        assert graph_sets(name).n_nodes == 200 and graph_sets(name).n_alloc == 64


def test_p10_statistics(graph_sets):
    gs = graph_sets("all10")
    frac = gs.node_perm.mean()
    assert abs(frac - 0.090) <= 0.005, frac  # 9.0% of kernels own permanent buffers
    perm_allocs = (gs.alloc_kind == 6).sum()
    assert perm_allocs == 2 * gs.node_perm.sum()  # "two permanent buffers" each
    assert (gs.allocs["size"][gs.alloc_kind == 6] == 512).all() and (gs.allocs["t_free"][gs.alloc_kind == 6] == T_NEVER).all()
    # 69.2% of a bs=1 Llama2-13B graph's kernels resolve through dlsym (calibration, +-6%)
    g13 = graph_sets("llama2-13b")
    sel = g13.node_bs == 1
    dl = (g13.func_kind[g13.func_id[sel]] == 0).mean()
    assert abs(dl - 0.692) < 0.06, dl


# ---------------------------------------------------------------- P11
def test_p11_r1_vs_r2_differ_only_on_dead_memory(graph_sets):
    gs = graph_sets("toy")
    a = as_tuples(gs.allocs)
    off = gs.node_word_off.tolist()
    r1 = brute.materialize(gs.words, off, gs.node_t.tolist(), a, "R1")
    r2 = brute.materialize(gs.words, off, gs.node_t.tolist(), a, "R2")
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    assert _slots_dict(m) == r2
    diff = {g for g in set(r1) | set(r2) if r1.get(g) != r2.get(g)}
    assert diff, "the toy set must exercise dangling words"
    for g in diff:
        assert gs.tags[g] in (TAG_DANGLING, TAG_OPE)
        assert g in r1 and g not in r2  # R1 relocates a word into freed memory; R2 leaves it constant
    for g in np.flatnonzero(gs.tags == TAG_DANGLING):
        assert int(g) in diff


# ---------------------------------------------------------------- P12
def test_p12_validation_counters_and_first_indices(graph_sets):
    gs = graph_sets("toy")
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    g, i, o = m["slot_g"].copy(), m["slot_id"].copy(), m["slot_off"].copy()
    src = gs.words.copy()
    new_size = gs.new_size.copy()
    table = gs.table.copy()
    fid = gs.func_id.copy()
    # STALE: the image word changed since materialization
    src[g[5]] ^= np.uint64(8)
    src[g[40]] ^= np.uint64(8)
    # BAD_ID: record points past the replayed allocation count
    i[10] = gs.n_alloc + 3
    # OOR: the replayed allocation shrank below the offset
    k = int(np.flatnonzero(o > 0)[3])
    new_size[i[k]] = o[k]
    # UNRESOLVED kernels
    table[fid[7]] = 0
    fid[3] = table.size + 1
    dst, fout, rep = oracle.restore(src, g, i, o, gs.allocs["base"], gs.new_base, new_size, fid, table)
    bd, bf, brep = brute.restore(src, {int(a): (int(b), int(c)) for a, b, c in zip(g, i, o)},
                                 gs.allocs["base"].tolist(), gs.new_base.tolist(), new_size.tolist(),
                                 fid.tolist(), table.tolist())
    assert [int(x) for x in dst] == bd and [int(x) for x in fout] == bf
    names = oracle.REPORT_FIELDS
    for q, nm in enumerate(names[:-1]):
        assert int(rep[q]) == brep[nm], nm
    n_oor = int(((o >= new_size[np.minimum(i, gs.n_alloc - 1)]) & (i < gs.n_alloc)).sum())
    assert rep[2] == 1 and rep[3] == n_oor >= 1 and rep[4] == 2
    assert rep[0] == rep[2] + rep[3] + rep[4]
    assert rep[1] == min(int(g[5]), int(g[10]), int(g[k]))
    assert rep[5] == int((fid == fid[7]).sum()) + 1 and rep[6] == min(3, int(np.flatnonzero(fid == fid[7])[0]))
    for bad_g in (g[5], g[10], g[40]):
        assert dst[bad_g] == src[bad_g]  # failed slots keep the source word


def test_pack_layout(graph_sets):
    gs = graph_sets("toy")
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    mask, cb, rec = oracle.pack(m, gs.n_words)
    bits = np.unpackbits(mask.view(np.uint8), bitorder="little")[: gs.n_words]
    assert np.array_equal(bits.astype(bool), m["is_slot"].astype(bool))
    assert cb[0] == 0 and cb[-1] == m["n_slots"]
    for c in range(cb.size - 1):
        assert cb[c] == m["is_slot"][: c * 2048].sum()
    assert np.array_equal(rec >> np.uint64(40), m["slot_id"].astype(np.uint64))
    assert np.array_equal(rec & np.uint64((1 << 40) - 1), m["slot_off"])
