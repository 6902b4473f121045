"""GPU restore driven by consistent and inconsistent packed tables (DESIGN.md
R-TABLE) against oracle.restore_packed, bit-exact: words, kernel addresses and
the report (incl. n_bad_chunk).  Both restore grids (one chunk per CTA for a
single model's set, two for the ten-model set), out of place, in place and
through the 8-byte-aligned scalar path."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU-only hosts
    pytest.skip("needs a GPU", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_asplos_zengxgcl25_b200 as medusa  # noqa: E402
from tests.test_oracle_table import _fixture_case, load_fixture  # noqa: E402

DEV = torch.device("cuda:0")


def _t(a):
    a = np.ascontiguousarray(a)
    dt = {8: np.int64, 4: np.int32}[a.dtype.itemsize]
    return torch.from_numpy(a.view(dt)).to(DEV)


def _gpu(src, mask, cb, rec, n_slots, ob, nb, ns, func_id=None, table=None, mode="out"):
    slots = medusa.Slots(_t(mask), _t(cb), _t(rec if rec.size else np.zeros(1, np.uint64)), n_slots)
    if table is not None:
        medusa.kernel_table_set(_t(table))
    s = _t(src)
    if mode == "in":
        dst, fout, rep = medusa.restore(s, slots, _t(ob), _t(nb), _t(ns), _t(func_id) if func_id is not None else None,
                                        dst=s)
    elif mode == "misaligned":
        big = torch.zeros(src.size + 1, dtype=torch.int64, device=DEV)
        big[1:] = s
        out = torch.zeros(src.size + 1, dtype=torch.int64, device=DEV)
        dst, fout, rep = medusa.restore(big[1:], slots, _t(ob), _t(nb), _t(ns),
                                        _t(func_id) if func_id is not None else None, dst=out[1:])
    else:
        dst, fout, rep = medusa.restore(s, slots, _t(ob), _t(nb), _t(ns), _t(func_id) if func_id is not None else None)
    torch.cuda.synchronize()
    return (medusa.to_numpy_u64(dst), medusa.to_numpy_u64(fout) if fout is not None else None,
            medusa.report_numpy(rep))


def _compare(src, mask, cb, rec, n_slots, ob, nb, ns, func_id=None, table=None):
    od, of, orp = oracle.restore_packed(src, mask, cb, rec, n_slots, ob, nb, ns, func_id, table)
    for mode in ("out", "in", "misaligned"):
        d, f, r = _gpu(src, mask, cb, rec, n_slots, ob, nb, ns, func_id, table, mode)
        assert np.array_equal(d, od), mode
        if func_id is not None:
            assert np.array_equal(f, of), mode
        assert np.array_equal(r, orp), (mode, r, orp)
    return orp


def test_hand_derived_fixture():
    fx = load_fixture()
    for case in fx["cases"]:
        src, mask, cb, rec, ns, allocs, nb, exp, rep = _fixture_case(fx, case)
        r = _compare(src, mask, cb, rec, ns, allocs["base"], nb, allocs["size"])
        assert np.array_equal(r, rep), case["what"]


@pytest.mark.parametrize("name", ["llama2-13b", "all10"])  # one chunk per restore CTA / two
def test_inconsistent_and_truncated_tables(graph_sets, name):
    gs = graph_sets(name)
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    mask, cb, rec = oracle.pack(m, gs.words.size)
    args = (gs.allocs["base"], gs.new_base, gs.new_size, gs.func_id, gs.table)
    # the caller's slot count cuts the table: the rest are missing records
    r = _compare(gs.words, mask, cb, rec, m["n_slots"] - 1000, *args)
    assert r[2] == 1000 and r[7] == 0
    # chunk_base corrupted at three places (each makes two neighbouring chunks
    # inconsistent, or one chunk decreasing), a mask bit set on a constant word,
    # a mask bit cleared on a slot word
    C = cb.size - 1
    cb2 = cb.copy()
    cb2[C // 3] += 1
    cb2[C // 2] = cb2[C // 2 - 1] - 1 if cb2[C // 2 - 1] > 0 else cb2[C // 2]
    cb2[C - 2] += 3
    mask2 = mask.copy()
    g_const = int(np.flatnonzero(m["is_slot"] == 0)[len(m["is_slot"]) // 5])
    mask2[g_const // 32] |= np.uint32(1 << (g_const % 32))
    g_slot = int(m["slot_g"][(2 * m["n_slots"]) // 3])
    mask2[g_slot // 32] &= np.uint32(~(1 << (g_slot % 32)) & 0xFFFFFFFF)
    r = _compare(gs.words, mask2, cb2, rec, m["n_slots"], *args)
    assert 4 <= r[7] <= 8
    # both at once, and a stale word
    src = gs.words.copy()
    src[int(m["slot_g"][17])] ^= np.uint64(64)
    r = _compare(src, mask2, cb2, rec, m["n_slots"] - 333, *args)
    assert r[2] >= 1 and r[7] >= 4


def test_bits_past_the_image_are_ignored(graph_sets):
    gs = graph_sets("toy")
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    n = (gs.words.size // 32) * 32 - 5  # a ragged last mask word
    mm = {k: v for k, v in m.items()}
    keep = m["slot_g"] < n
    mm.update(is_slot=m["is_slot"][:n], id=m["id"][:n], off=m["off"][:n], n_slots=int(keep.sum()),
              slot_g=m["slot_g"][keep], slot_id=m["slot_id"][keep], slot_off=m["slot_off"][keep])
    mask, cb, rec = oracle.pack(mm, n)
    mask[-1] |= np.uint32(0xFFFFFFFF ^ ((1 << (n % 32)) - 1)) if n % 32 else np.uint32(0)
    r = _compare(gs.words[:n], mask, cb, rec, mm["n_slots"], gs.allocs["base"], gs.new_base, gs.new_size)
    assert r[0] == 0 and r[7] == 0
