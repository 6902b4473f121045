"""The seeded input generator: determinism, well-formedness, shapes, replication."""
import numpy as np
import pytest

import oracle
from workloads import ALLOC_DTYPE, TAG_CONST, make_graph_set
from workloads.graphset import replicate


def test_deterministic(graph_sets):
    a = make_graph_set("toy")
    b = make_graph_set("toy")
    for k in ("words", "node_word_off", "node_t", "func_id", "new_base", "table", "tags"):
        assert np.array_equal(getattr(a, k), getattr(b, k)), k
    assert np.array_equal(a.allocs, b.allocs)
    c = make_graph_set("toy", seed=2)
    assert not np.array_equal(a.words, c.words)


@pytest.mark.parametrize("name", ["toy", "qwen1.5-4b", "llama2-7b", "llama2-13b", "all10"])
def test_configs_are_well_formed_and_shaped(graph_sets, name):
    gs = graph_sets(name)
    assert gs.allocs.dtype == ALLOC_DTYPE and gs.allocs.itemsize == 24
    assert oracle.check(gs.n_words, gs.node_word_off, gs.node_t, gs.allocs) == oracle.OK
    assert (np.diff(gs.node_t.astype(np.int64)) > 0).all()
    assert int(gs.node_word_off[-1]) == gs.n_words
    assert gs.func_id.max() < gs.table.size and (gs.table != 0).all()
    assert (gs.new_size == gs.allocs["size"]).all()
    # bytes per node ~ 175-190, toy excepted
    if name != "toy":
        assert 165 <= gs.n_words * 8 / gs.n_nodes <= 195


def test_replicate_is_r_shifted_copies(graph_sets):
    gs = graph_sets("toy")
    big = replicate(gs, 3)
    assert big.n_words == 3 * gs.n_words and big.n_alloc == 3 * gs.n_alloc and big.n_nodes == 3 * gs.n_nodes
    m1 = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    m3 = oracle.materialize(big.words, big.node_word_off, big.node_t, big.allocs)
    assert m3["status"] == 0 and m3["n_slots"] == 3 * m1["n_slots"]
    for r in range(3):
        sl = slice(r * gs.n_words, (r + 1) * gs.n_words)
        assert np.array_equal(m3["is_slot"][sl], m1["is_slot"])
        assert np.array_equal(m3["id"][sl][m1["is_slot"] == 1], m1["id"][m1["is_slot"] == 1] + r * gs.n_alloc)
        assert np.array_equal(m3["off"][sl], m1["off"])
    consts = gs.tags == TAG_CONST
    assert np.array_equal(big.words[gs.n_words:2 * gs.n_words][consts], gs.words[consts])


def test_inband_stress_config(graph_sets):
    """all10-inband: the ten-model set (Table 1 totals kept) with 5-10% of all words
    in-band non-pointer constants -- inside [least base, greatest end) of the
    trace, so the classify prefilter passes them -- and still well-formed."""
    gs = graph_sets("all10-inband")
    assert gs.n_nodes == 139364
    assert oracle.check(gs.n_words, gs.node_word_off, gs.node_t, gs.allocs) == oracle.OK
    a = gs.allocs
    live = a["size"] > 0
    lo, hi = a["base"][live].min(), (a["base"][live] + a["size"][live]).max()
    inband = (gs.words >= lo) & (gs.words < hi)
    frac = float((inband & (gs.tags != 1)).mean())
    assert 0.05 <= frac <= 0.10, frac
