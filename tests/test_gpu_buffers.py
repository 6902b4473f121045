"""GPU parity of copy-free buffer contents restoration (§4.3,
P:218-224) through the C ABI against oracle/buffers.py, bit-exact: the class
of every allocation, the permanent-buffer list and blob layout, the saved blob,
every byte of the replayed memory after restore, and the report."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU-only hosts
    pytest.skip("needs a GPU", allow_module_level=True)

import oracle  # noqa: E402
from oracle import buffers as ob  # noqa: E402
import paper_conf_asplos_zengxgcl25_b200 as medusa  # noqa: E402
from workloads import ALLOC_DTYPE, T_NEVER  # noqa: E402

DEV = torch.device("cuda:0")
NONE = (1 << 64) - 1


def _h(t):
    return t.detach().cpu().numpy()


def _plan_check(plan, cls, perm, off):
    assert np.array_equal(_h(plan.cls), cls)
    assert plan.n_perm == perm.size
    assert np.array_equal(_h(plan.perm).view(np.uint32), perm)
    assert np.array_equal(_h(plan.perm_off).view(np.uint64), off)
    assert plan.blob_bytes == int(off[-1])


@pytest.mark.parametrize("name", ["toy", "qwen1.5-4b", "llama2-7b", "all10"])
def test_plan_parity(graph_sets, name):
    gs = graph_sets(name)
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    plan = medusa.buffers_plan(inp["allocs"], inp["capture_t"], slots.slot, slots.n_slots)
    torch.cuda.synchronize()
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    cls = ob.classify(gs.allocs, gs.capture_t, m["slot_id"])
    perm, off = ob.plan(gs.allocs, cls)
    _plan_check(plan, cls, perm, off)
    assert plan.n_perm == 2 * int(gs.node_perm.sum())


def _real_case(seed, n=300, n_cap=3):
    """A trace whose allocations live in a real device arena (old run) and are
    replayed into a second arena in another order (online run): sizes include
    0, odd and large; bases include non-16-byte-aligned ones."""
    rng = np.random.default_rng(seed)
    sizes = rng.choice([0, 1, 4, 13, 16, 100, 512, 4096, 70000], size=n,
                       p=[.03, .05, .2, .07, .1, .1, .3, .1, .05]).astype(np.int64)
    pad = rng.choice([0, 1, 8, 16, 512], size=n)
    old_pos = np.concatenate([[0], np.cumsum(sizes + pad)[:-1]])
    order = rng.permutation(n)
    new_pos = np.zeros(n, np.int64)
    cur = 0
    for i in order:
        new_pos[i] = cur
        cur += int(sizes[i]) + int(rng.choice([0, 3, 16]))
    old_arena = torch.randint(0, 256, (int(old_pos[-1] + sizes[-1] + 64),), dtype=torch.uint8, device=DEV)
    new_arena = torch.full((cur + 64,), 0xA5, dtype=torch.uint8, device=DEV)
    a = np.zeros(n, ALLOC_DTYPE)
    a["base"] = (old_arena.data_ptr() + old_pos).astype(np.uint64)
    a["size"] = sizes.astype(np.uint64)
    # events: capture k spans ordinals [k*n/(n_cap+1) + n/(2(n_cap+1)), ...): a mix of
    # before-capture, in-capture freed / never freed
    t = np.arange(n, dtype=np.int64) * 4 + 10
    a["t_alloc"] = t
    tf = np.where(rng.random(n) < 0.5, t + 2, T_NEVER)
    a["t_free"] = tf
    caps = []
    step = n // n_cap
    for k in range(n_cap):
        b = int(t[k * step + step // 4]) - 1
        e = int(t[k * step + 3 * step // 4]) + 1
        caps.append((b, e))
    capture_t = np.asarray(caps, np.uint32)
    ids = rng.choice(n, size=2 * n, replace=True)
    slot = (ids.astype(np.uint64) << np.uint64(40)) | rng.integers(0, 8, size=ids.size).astype(np.uint64)
    new_base = (new_arena.data_ptr() + new_pos).astype(np.uint64)
    return a, capture_t, slot, ids, old_arena, new_arena, new_base


def _dev(x, dt):
    return torch.from_numpy(np.ascontiguousarray(x).view(dt)).to(DEV)


@pytest.mark.parametrize("seed", range(4))
def test_save_restore_real_memory(seed):
    a, capture_t, slot, ids, old_arena, new_arena, new_base = _real_case(seed)
    d_allocs = _dev(a, np.int64).reshape(-1, 3)
    plan = medusa.buffers_plan(d_allocs, _dev(capture_t, np.int32), _dev(slot, np.int64), slot.size)
    blob, rep_s = medusa.buffers_save(plan, _dev(a["base"], np.int64))
    rep_r = medusa.buffers_restore(plan, blob, _dev(new_base, np.int64), _dev(a["size"], np.int64))
    torch.cuda.synchronize()
    cls = ob.classify(a, capture_t, ids)
    perm, off = ob.plan(a, cls)
    _plan_check(plan, cls, perm, off)
    assert (cls == ob.PERM).sum() > 20 and (cls == ob.TEMP).sum() > 20 and (cls == ob.PARAM).sum() > 20
    old = ob.Arena(old_arena.data_ptr(), data=_h(old_arena))
    exp_blob = ob.save(old, perm, off, a["base"])
    assert np.array_equal(_h(blob)[: exp_blob.size], exp_blob)
    new = ob.Arena(new_arena.data_ptr(), data=np.full(new_arena.numel(), 0xA5, np.uint8))
    assert ob.restore(new, exp_blob, perm, off, new_base, a["size"]) == (0, NONE)
    assert np.array_equal(_h(new_arena), new.data)
    assert _h(rep_s).view(np.uint64).tolist() == [0, NONE] == _h(rep_r).view(np.uint64).tolist()


def test_restore_faults_match_oracle():
    a, capture_t, slot, ids, old_arena, new_arena, new_base = _real_case(11)
    d_allocs = _dev(a, np.int64).reshape(-1, 3)
    plan = medusa.buffers_plan(d_allocs, _dev(capture_t, np.int32), _dev(slot, np.int64), slot.size)
    blob, _ = medusa.buffers_save(plan, _dev(a["base"], np.int64))
    cls = ob.classify(a, capture_t, ids)
    perm, off = ob.plan(a, cls)
    size = a["size"].copy()
    big = [int(i) for i in perm if size[i] > 0]
    size[big[1]] -= 1          # replayed allocation smaller than the saved one
    size[big[5]] = 0
    short = int(perm[-3])      # the replay made fewer allocations
    rep = medusa.buffers_restore(plan, blob, _dev(new_base[:short], np.int64), _dev(size[:short], np.int64))
    torch.cuda.synchronize()
    old = ob.Arena(old_arena.data_ptr(), data=_h(old_arena))
    new = ob.Arena(new_arena.data_ptr(), data=np.full(new_arena.numel(), 0xA5, np.uint8))
    n_bad, first = ob.restore(new, ob.save(old, perm, off, a["base"]), perm, off, new_base[:short], size[:short])
    assert n_bad == 5
    assert _h(rep).view(np.uint64).tolist() == [n_bad, first]
    assert np.array_equal(_h(new_arena), new.data)


def test_plan_errors_and_capacity():
    a, capture_t, slot, ids, *_ = _real_case(3)
    d_allocs = _dev(a, np.int64).reshape(-1, 3)
    d_slot = _dev(slot, np.int64)
    bad = capture_t.copy()
    bad[1, 0] = bad[0, 1] - 1  # overlapping captures
    with pytest.raises(medusa.MedusaError) as ei:
        medusa.buffers_plan(d_allocs, _dev(bad, np.int32), d_slot, slot.size)
    assert ei.value.status == medusa.ERR_INVALID_ARG
    cls = ob.classify(a, capture_t, ids)
    perm, off = ob.plan(a, cls)
    with pytest.raises(medusa.MedusaError) as ei:
        medusa.buffers_plan(d_allocs, _dev(capture_t, np.int32), d_slot, slot.size, capacity=perm.size - 1)
    assert ei.value.status == medusa.ERR_CAPACITY
    assert (ei.value.n_perm, ei.value.blob_bytes) == (perm.size, int(off[-1]))
    # exact capacity succeeds; no captures -> everything referenced is PARAM, no blob
    plan = medusa.buffers_plan(d_allocs, _dev(capture_t, np.int32), d_slot, slot.size, capacity=perm.size)
    _plan_check(plan, cls, perm, off)
    plan = medusa.buffers_plan(d_allocs, torch.empty((0, 2), dtype=torch.int32, device=DEV), d_slot, slot.size)
    torch.cuda.synchronize()
    assert plan.n_perm == 0 and plan.blob_bytes == 0
    assert np.array_equal(_h(plan.cls), ob.classify(a, np.zeros((0, 2)), ids))
    blob, rep = medusa.buffers_save(plan, _dev(a["base"], np.int64))
    rep2 = medusa.buffers_restore(plan, blob, _dev(a["base"], np.int64), _dev(a["size"], np.int64))
    torch.cuda.synchronize()
    assert _h(rep).view(np.uint64).tolist() == [0, NONE] == _h(rep2).view(np.uint64).tolist()


def test_all10_save_restore_full_size(graph_sets):
    """Full ten-model set: the plan from the GPU table, then the PERM buffers given
    real addresses (an arena, 512-B apart, replayed in shuffled order) and saved /
    restored in the launch configuration bench.py times."""
    gs = graph_sets("all10")
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    plan = medusa.buffers_plan(inp["allocs"], inp["capture_t"], slots.slot, slots.n_slots)
    torch.cuda.synchronize()
    perm = _h(plan.perm).view(np.uint32)
    sizes = gs.allocs["size"][perm].astype(np.int64)
    rng = np.random.default_rng(4)
    old_arena = torch.randint(0, 256, (int(sizes.sum()),), dtype=torch.uint8, device=DEV)
    new_arena = torch.full((int(sizes.sum()),), 0x5A, dtype=torch.uint8, device=DEV)
    base = np.zeros(gs.n_alloc, np.uint64)
    nb = np.zeros(gs.n_alloc, np.uint64)
    pos = np.concatenate([[0], np.cumsum(sizes)[:-1]])
    base[perm] = old_arena.data_ptr() + pos
    sh = rng.permutation(perm.size)
    nb[perm[sh]] = new_arena.data_ptr() + pos
    blob, rep_s = medusa.buffers_save(plan, _dev(base, np.int64))
    rep_r = medusa.buffers_restore(plan, blob, _dev(nb, np.int64), _dev(gs.new_size, np.int64))
    torch.cuda.synchronize()
    assert _h(rep_s).view(np.uint64).tolist() == [0, NONE] == _h(rep_r).view(np.uint64).tolist()
    assert np.array_equal(_h(blob), _h(old_arena))  # arena order == ordinal order
    old, new = _h(old_arena), _h(new_arena)
    for k in rng.choice(perm.size, size=500, replace=False):  # sampled buffers, one by one
        i = perm[k]
        s = int(sizes[k])
        o = int(base[i]) - old_arena.data_ptr()
        n = int(nb[i]) - new_arena.data_ptr()
        assert np.array_equal(new[n:n + s], old[o:o + s])
    assert np.array_equal(np.sort(new), np.sort(old))
