"""Pins of oracle.restore_packed (DESIGN.md R-TABLE: restore driven by the packed
table, consistent or not), no GPU.

* on every table oracle_pack_slots writes (always consistent), the packed
  restoration equals the logical one (oracle.restore over the slot list) --
  toy and Qwen-shaped sets, tiny adversarial traces, injected faults, a caller
  slot count that cuts the table;
* a hand-derived fixture (tests/golden/table_consistency.json) fixes the
  inconsistent cases: extra / missing records per chunk, a decreasing range,
  bits past n_words.
"""
import json
import os

import numpy as np
import pytest

import oracle
from tests.tiny import tiny_trace
from workloads import ALLOC_DTYPE

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
MAX = np.uint64(2**64 - 1)


def _both(words, m, old_base, new_base, new_size, func_id=None, table=None, n_slots=None):
    mask, cb, rec = oracle.pack(m, words.size)
    ns = m["n_slots"] if n_slots is None else n_slots
    a = oracle.restore_packed(words, mask, cb, rec, ns, old_base, new_base, new_size, func_id, table)
    k = ns
    b = oracle.restore(words, m["slot_g"][:k], m["slot_id"][:k], m["slot_off"][:k], old_base, new_base, new_size,
                       func_id, table)
    return a, b


@pytest.mark.parametrize("name", ["toy", "qwen1.5-4b"])
def test_packed_equals_logical_on_generated_sets(graph_sets, name):
    gs = graph_sets(name)
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    (d1, f1, r1), (d2, f2, r2) = _both(gs.words, m, gs.allocs["base"], gs.new_base, gs.new_size, gs.func_id, gs.table)
    assert np.array_equal(d1, d2) and np.array_equal(f1, f2) and np.array_equal(r1, r2)
    assert r1[7] == 0 and r1[0] == 0


def test_packed_equals_logical_with_faults(graph_sets):
    gs = graph_sets("toy")
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    src = gs.words.copy()
    src[m["slot_g"][3]] ^= np.uint64(8)
    ns = gs.new_size.copy()
    ns[m["slot_id"][10]] = 0
    n_rep = int(m["slot_id"].max())
    (d1, _, r1), (d2, _, r2) = _both(src, m, gs.allocs["base"][:n_rep], gs.new_base[:n_rep], ns[:n_rep])
    assert np.array_equal(d1, d2) and np.array_equal(r1, r2)
    assert r1[2] > 0 and r1[3] > 0 and r1[4] > 0


def test_truncated_slot_count_is_missing_records(graph_sets):
    """n_slots below the table total: the slots past it keep their words and count
    as bad ids -- the logical restoration of the remaining slots plus those."""
    gs = graph_sets("toy")
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    cut = m["n_slots"] - 37
    mask, cb, rec = oracle.pack(m, gs.words.size)
    d1, _, r1 = oracle.restore_packed(gs.words, mask, cb, rec, cut, gs.allocs["base"], gs.new_base, gs.new_size)
    d2, _, r2 = oracle.restore(gs.words, m["slot_g"][:cut], m["slot_id"][:cut], m["slot_off"][:cut],
                               gs.allocs["base"], gs.new_base, gs.new_size)
    assert np.array_equal(d1, d2)  # the missing slots keep their source words
    assert r1[0] == 37 and r1[2] == 37 and r1[1] == m["slot_g"][cut] and r1[7] == 0


def test_packed_equals_logical_on_tiny_traces():
    seen = 0
    for seed in range(150):
        words, off, nt, allocs = tiny_trace(5000 + seed, n_steps=400, max_words=40, max_allocs=80)
        m = oracle.materialize(words, off, nt, allocs)
        if m["status"] != 0:
            continue
        rng = np.random.default_rng(seed)
        new_base = allocs["base"] + rng.integers(0, 1 << 30, allocs.size, dtype=np.uint64) * np.uint64(16)
        (d1, _, r1), (d2, _, r2) = _both(words, m, allocs["base"], new_base, allocs["size"])
        assert np.array_equal(d1, d2) and np.array_equal(r1, r2), seed
        seen += words.size > 2048
    assert seen > 0  # some traces span several chunks


def _fixture_case(fx, case):
    n = fx["n_words"]
    src = np.zeros(n, np.uint64)
    for g, v in fx["src_nonzero"].items():
        src[int(g)] = int(v, 16)
    mask = np.zeros((n + 31) // 32, np.uint32)
    for g in fx["mask_bits"]:
        mask[g // 32] |= np.uint32(1 << (g % 32))
    rec = np.array([int(x, 16) for x in fx["records"]], np.uint64)
    for k, v in case.get("records_override", {}).items():
        rec[int(k)] = int(v, 16)
    allocs = np.zeros(len(fx["allocs"]), ALLOC_DTYPE)
    for i, (b, s) in enumerate(fx["allocs"]):
        allocs[i] = (int(b, 16), int(s, 16), i + 1, 0xFFFFFFFF)
    new_base = np.array([int(x, 16) for x in fx["new_base"]], np.uint64)
    exp = src.copy()
    for g, v in case["dst_changed"].items():
        exp[int(g)] = int(v, 16)
    rep = np.array([MAX if x == "max" else x for x in case["report"]], np.uint64)
    return src, mask, np.array(case["chunk_base"], np.uint32), rec, case["n_slots"], allocs, new_base, exp, rep


def load_fixture():
    return json.load(open(os.path.join(GOLDEN, "table_consistency.json")))


def test_hand_derived_inconsistent_tables():
    fx = load_fixture()
    for case in fx["cases"]:
        src, mask, cb, rec, ns, allocs, nb, exp, rep = _fixture_case(fx, case)
        dst, _, r = oracle.restore_packed(src, mask, cb, rec, ns, allocs["base"], nb, allocs["size"])
        assert np.array_equal(dst, exp), case["what"]
        assert np.array_equal(r, rep), (case["what"], r)
