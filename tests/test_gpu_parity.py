"""GPU parity: the CUDA path (through the C ABI) against the oracle, bit-exact.

Every comparison is element by element on the same seeded inputs: the
materialized table (mask, chunk prefix, records), the restored words, the
kernel-address fill and the report.  Sizes: the toy set and the three
single-model BASELINE configs in full, the ten-model set (139,364 nodes) in
full, in the launch configuration bench.py times.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU-only hosts
    pytest.skip("needs a GPU", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_asplos_zengxgcl25_b200 as medusa  # noqa: E402
from tests.tiny import tiny_trace  # noqa: E402
from workloads import ALLOC_DTYPE, T_NEVER  # noqa: E402

DEV = torch.device("cuda:0")


def _h(t):
    return t.detach().cpu().numpy()


def _oracle_full(words, node_off, node_t, allocs, new_base, new_size, func_id=None, table=None):
    m = oracle.materialize(words, node_off, node_t, allocs)
    if m["status"] != 0:
        return m, None
    mask, cb, rec = oracle.pack(m, words.size)
    dst, fout, rep = oracle.restore(words, m["slot_g"], m["slot_id"], m["slot_off"], allocs["base"], new_base,
                                    new_size, func_id, table)
    return m, (mask, cb, rec, dst, fout, rep)


def _check_materialize(slots, m, packed, n_words):
    mask, cb, rec = packed[:3]
    assert slots.n_slots == m["n_slots"]
    assert np.array_equal(_h(slots.mask).view(np.uint32), mask)
    assert np.array_equal(_h(slots.chunk_base).view(np.uint32), cb)
    assert np.array_equal(_h(slots.slot[:slots.n_slots]).view(np.uint64), rec)


@pytest.mark.parametrize("name", ["toy", "qwen1.5-4b", "llama2-7b", "llama2-13b", "all10", "all10-inband"])
def test_full_path_parity(graph_sets, name):
    gs = graph_sets(name)
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    medusa.kernel_table_set(inp["table"])
    dst, fout, rep = medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"],
                                    inp["func_id"])
    torch.cuda.synchronize()
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size,
                             gs.func_id, gs.table)
    assert m["status"] == 0
    _check_materialize(slots, m, packed, gs.n_words)
    assert np.array_equal(medusa.to_numpy_u64(dst), packed[3])
    assert np.array_equal(medusa.to_numpy_u64(fout), packed[4])
    assert np.array_equal(medusa.report_numpy(rep), packed[5])
    assert medusa.report_numpy(rep)[0] == 0


def test_restore_driven_by_oracle_table(graph_sets):
    """K3+K4 in isolation: the oracle's packed table fed to the GPU restore."""
    gs = graph_sets("llama2-7b")
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size,
                             gs.func_id, gs.table)
    mask, cb, rec, dst_o, fout_o, rep_o = packed
    inp = medusa.upload(gs, DEV)
    slots = medusa.Slots(torch.from_numpy(mask.view(np.int32)).to(DEV), torch.from_numpy(cb.view(np.int32)).to(DEV),
                         torch.from_numpy(rec.view(np.int64)).to(DEV), m["n_slots"])
    medusa.kernel_table_set(inp["table"])
    dst, fout, rep = medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"],
                                    inp["func_id"])
    assert np.array_equal(medusa.to_numpy_u64(dst), dst_o)
    assert np.array_equal(medusa.to_numpy_u64(fout), fout_o)
    assert np.array_equal(medusa.report_numpy(rep), rep_o)


@pytest.mark.parametrize("name", ["qwen1.5-4b", "all10"])  # one chunk per restore CTA / two
def test_in_place_and_misaligned(graph_sets, name):
    gs = graph_sets(name)
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size)
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    buf = inp["words"].clone()
    dst, _, rep = medusa.restore(buf, slots, inp["old_base"], inp["new_base"], inp["new_size"], dst=buf)
    assert dst.data_ptr() == buf.data_ptr()
    assert np.array_equal(medusa.to_numpy_u64(buf), packed[3])
    # 8-byte but not 16-byte aligned image and output: scalar path, same bytes
    big = torch.zeros(gs.n_words + 1, dtype=torch.int64, device=DEV)
    big[1:] = inp["words"]
    out = torch.zeros(gs.n_words + 1, dtype=torch.int64, device=DEV)
    src_v, dst_v = big[1:], out[1:]
    slots2 = medusa.materialize(src_v, inp["node_off"], inp["node_t"], inp["allocs"])
    _check_materialize(slots2, m, packed, gs.n_words)
    medusa.restore(src_v, slots2, inp["old_base"], inp["new_base"], inp["new_size"], dst=dst_v)
    assert np.array_equal(medusa.to_numpy_u64(dst_v), packed[3])


@pytest.mark.parametrize("name", ["toy", "all10"])
def test_in_place_full_path(graph_sets, name):
    """In-place restore (the online phase patches the loaded image) at full size:
    bit-exact restored image, kernel-address fill and report."""
    gs = graph_sets(name)
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    medusa.kernel_table_set(inp["table"])
    buf = inp["words"].clone()
    _, fout, rep = medusa.restore(buf, slots, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                                  dst=buf)
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size,
                             gs.func_id, gs.table)
    assert np.array_equal(medusa.to_numpy_u64(buf), packed[3])
    assert np.array_equal(medusa.to_numpy_u64(fout), packed[4])
    assert np.array_equal(medusa.report_numpy(rep), packed[5])


@pytest.mark.parametrize("name", ["toy", "llama2-13b"])
def test_restore_writes_every_word(graph_sets, name):
    """Every destination word is written (the kernel stores whole tiles with TMA
    bulk stores, which compute-sanitizer initcheck does not track): dst starts as
    two different sentinel fills and both runs end bit-identical to the oracle."""
    gs = graph_sets(name)
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size)
    for fill in (-1, 0x5A5A5A5A5A5A5A5A):
        dst = torch.full_like(inp["words"], fill)
        medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"], dst=dst)
        assert np.array_equal(medusa.to_numpy_u64(dst), packed[3]), fill


def test_fault_injection_matches_oracle(graph_sets):
    gs = graph_sets("toy")
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    g = m["slot_g"]
    src = gs.words.copy()
    src[g[5]] ^= np.uint64(8)  # STALE
    src[g[33]] ^= np.uint64(16)
    new_size = gs.new_size.copy()
    k = int(np.flatnonzero(m["slot_off"] > 0)[2])
    new_size[m["slot_id"][k]] = m["slot_off"][k]  # OOR for every slot of that allocation at off >= size
    table = gs.table.copy()
    table[gs.func_id[7]] = 0  # unresolved kernels
    fid = gs.func_id.copy()
    fid[3] = table.size + 5
    n_alloc_replay = int(m["slot_id"].max())  # the last allocation(s) missing from the replay: BAD_ID
    ob, nb, ns = gs.allocs["base"][:n_alloc_replay], gs.new_base[:n_alloc_replay], new_size[:n_alloc_replay]
    dst_o, fout_o, rep_o = oracle.restore(src, m["slot_g"], m["slot_id"], m["slot_off"], ob, nb, ns, fid, table)
    assert rep_o[2] > 0 and rep_o[3] > 0 and rep_o[4] == 2 and rep_o[5] > 0
    t = lambda a, dt=torch.int64: torch.from_numpy(np.ascontiguousarray(a).view(np.int64 if dt == torch.int64 else np.int32)).to(DEV)
    medusa.kernel_table_set(t(table))
    dst, fout, rep = medusa.restore(t(src), slots, t(ob), t(nb), t(ns), t(fid, torch.int32))
    assert np.array_equal(medusa.to_numpy_u64(dst), dst_o)
    assert np.array_equal(medusa.to_numpy_u64(fout), fout_o)
    assert np.array_equal(medusa.report_numpy(rep), rep_o)
    # the same faults in place (dst == src: only slot words are read and written)
    buf = t(src)
    dst_i, fout_i, rep_i = medusa.restore(buf, slots, t(ob), t(nb), t(ns), t(fid, torch.int32), dst=buf)
    assert dst_i.data_ptr() == buf.data_ptr()
    assert np.array_equal(medusa.to_numpy_u64(buf), dst_o)
    assert np.array_equal(medusa.to_numpy_u64(fout_i), fout_o)
    assert np.array_equal(medusa.report_numpy(rep_i), rep_o)
    # the report is rewritten completely by the next call
    medusa.kernel_table_set(inp["table"])
    _, _, rep2 = medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"],
                                inp["func_id"])
    r2 = medusa.report_numpy(rep2)
    assert r2[0] == 0 and r2[1] == np.uint64(2**64 - 1) and r2[5] == 0 and r2[7] == 0


def _run_tiny(words, off, node_t, allocs):
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(DEV)
    aa = np.ascontiguousarray(allocs).view(np.int64).reshape(-1, 3) if allocs.size else np.zeros((0, 3), np.int64)
    try:
        s = medusa.materialize(t(words, np.int64), t(off, np.int64), t(node_t, np.int32),
                               torch.from_numpy(aa).to(DEV))
        return 0, s
    except medusa.MedusaError as e:
        return e.status, None


@pytest.mark.parametrize("overlap_p", [0.0, 0.2])
def test_tiny_traces_status_and_slots(overlap_p):
    """Adversarial tiny traces (reuse, adjacency, zero sizes, equal positions,
    empty nodes, malformed traces): status and table identical to the oracle."""
    for seed in range(300):
        words, off, node_t, allocs = tiny_trace(seed * 7 + int(overlap_p * 1000), overlap_p=overlap_p)
        st, s = _run_tiny(words, off, node_t, allocs)
        m = oracle.materialize(words, off, node_t, allocs)
        assert st == m["status"], (seed, st, m["status"])
        if st == 0:
            mask, cb, rec = oracle.pack(m, words.size)
            assert s.n_slots == m["n_slots"]
            assert np.array_equal(_h(s.mask).view(np.uint32), mask), seed
            assert np.array_equal(_h(s.chunk_base).view(np.uint32), cb), seed
            assert np.array_equal(_h(s.slot[:s.n_slots]).view(np.uint64), rec), seed


@pytest.mark.parametrize("seed", range(6))
def test_long_chunks_many_nodes_and_window_batches(seed):
    """Chunks holding ~1000 nodes (several live-mask node groups) whose windows
    hold hundreds of registered mortals (several window batches), with heavy
    address reuse: status and table identical to the oracle."""
    words, off, node_t, allocs = tiny_trace(1000 + seed, n_steps=7000, max_words=2, max_allocs=2500,
                                            overlap_p=0.0 if seed < 5 else 0.01)
    st, s = _run_tiny(words, off, node_t, allocs)
    m = oracle.materialize(words, off, node_t, allocs)
    assert st == m["status"]
    assert words.size > 2048 and node_t.size > 2000 and allocs.size > 1000
    if st == 0:
        mask, cb, rec = oracle.pack(m, words.size)
        assert s.n_slots == m["n_slots"]
        assert np.array_equal(_h(s.mask).view(np.uint32), mask)
        assert np.array_equal(_h(s.chunk_base).view(np.uint32), cb)
        assert np.array_equal(_h(s.slot[:s.n_slots]).view(np.uint64), rec)


def test_edge_cases():
    b = 0x7F00_0000_0000
    A = lambda rows: np.array(rows, dtype=ALLOC_DTYPE)
    # empty image, no nodes
    st, s = _run_tiny(np.zeros(0, np.uint64), np.zeros(1, np.uint64), np.zeros(0, np.uint32), A([]))
    assert st == 0 and s.n_slots == 0 and _h(s.chunk_base)[0] == 0
    # nodes but no words; allocations but no words
    st, s = _run_tiny(np.zeros(0, np.uint64), np.zeros(4, np.uint64), np.array([3, 5, 9], np.uint32),
                      A([(b, 64, 1, T_NEVER)]))
    assert st == 0 and s.n_slots == 0
    # no allocations: everything is a constant
    w = np.arange(5000, dtype=np.uint64) + np.uint64(b)
    st, s = _run_tiny(w, np.array([0, 4999, 5000], np.uint64), np.array([1, 2], np.uint32), A([]))
    assert st == 0 and s.n_slots == 0
    # one allocation covering a ragged multi-chunk image: every word a slot
    w = np.uint64(b) + np.arange(5000, dtype=np.uint64) * np.uint64(8)
    st, s = _run_tiny(w, np.array([0, 1, 4096, 5000], np.uint64), np.array([2, 3, 4], np.uint32),
                      A([(b, 8 * 5000, 1, T_NEVER)]))
    assert st == 0 and s.n_slots == 5000
    assert (_h(s.slot[:5000]) == np.arange(5000) * 8).all()
    # a single node spanning many chunks with its allocation freed before it launches
    st, s = _run_tiny(w, np.array([0, 5000], np.uint64), np.array([9], np.uint32), A([(b, 8 * 5000, 1, 9)]))
    assert st == 0 and s.n_slots == 0
    # invalid arguments detected on the device
    st, _ = _run_tiny(w[:4], np.array([0, 3, 2, 4], np.uint64), np.array([1, 2, 3], np.uint32), A([]))
    assert st == medusa.ERR_INVALID_ARG
    st, _ = _run_tiny(w[:4], np.array([0, 2, 4], np.uint64), np.array([2, 2], np.uint32), A([]))
    assert st == medusa.ERR_INVALID_ARG
    st, _ = _run_tiny(w[:4], np.array([0, 4], np.uint64), np.array([2], np.uint32), A([(b, (1 << 40) + 8, 1, 3)]))
    assert st == medusa.ERR_INVALID_ARG
    st, _ = _run_tiny(w[:4], np.array([0, 4], np.uint64), np.array([2], np.uint32), A([(b, 64, 3, 3)]))
    assert st == medusa.ERR_TRACE


def test_no_allocations_after_a_large_call(graph_sets):
    """The allocation-free path (no k_prepare between k_trace and k_classify) right
    after a ten-model call left its chunk / node scratch behind: nothing but
    constants, no stale node range used."""
    gs = graph_sets("all10")
    inp = medusa.upload(gs, DEV)
    medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    n = gs.n_words // 3  # many chunks and nodes, all constants
    off = gs.node_word_off[: int(np.searchsorted(gs.node_word_off, n)) + 1].copy()
    off[-1] = n
    st, s = _run_tiny(gs.words[:n], off, gs.node_t[: off.size - 1], np.zeros(0, ALLOC_DTYPE))
    assert st == 0 and s.n_slots == 0
    assert not _h(s.mask).any() and not _h(s.chunk_base).any()


def test_capacity_too_small(graph_sets):
    gs = graph_sets("toy")
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    inp = medusa.upload(gs, DEV)
    with pytest.raises(medusa.MedusaError) as ei:
        medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], capacity=10)
    assert ei.value.status == medusa.ERR_CAPACITY and ei.value.n_slots == m["n_slots"]
    s = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], capacity=m["n_slots"])
    assert s.n_slots == m["n_slots"]


def test_multi_chunk_malformed_ten_model_trace(graph_sets):
    """A single overlapping allocation injected into the full ten-model trace is rejected."""
    gs = graph_sets("all10")
    allocs = gs.allocs.copy()
    i = int(np.flatnonzero(gs.alloc_kind == 5)[5000])  # a capture temporary
    j = i + 1
    while allocs["size"][j] == 0 or not (allocs["t_alloc"][j] < allocs["t_free"][i]):
        j += 1
    allocs["base"][j] = allocs["base"][i] + np.uint64(8)  # overlaps i while both live
    assert oracle.check(gs.n_words, gs.node_word_off, gs.node_t, allocs) == oracle.ERR_TRACE
    inp = medusa.upload(gs, DEV)
    aa = torch.from_numpy(np.ascontiguousarray(allocs).view(np.int64).reshape(-1, 3)).to(DEV)
    with pytest.raises(medusa.MedusaError) as ei:
        medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], aa)
    assert ei.value.status == medusa.ERR_TRACE


def test_replicated_multi_instance_parity(graph_sets):
    """Three replicas of the Llama-2-7B-shaped set in one call (ids up to 3 x n_alloc,
    3x the chunks): bit-exact against the oracle."""
    from workloads.graphset import replicate
    gs = replicate(graph_sets("llama2-7b"), 3)
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    medusa.kernel_table_set(inp["table"])
    dst, fout, rep = medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"],
                                    inp["func_id"])
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size,
                             gs.func_id, gs.table)
    _check_materialize(slots, m, packed, gs.n_words)
    assert np.array_equal(medusa.to_numpy_u64(dst), packed[3])
    assert np.array_equal(medusa.to_numpy_u64(fout), packed[4])
    assert np.array_equal(medusa.report_numpy(rep), packed[5])


@pytest.mark.parametrize("name", ["toy", "all10"])
def test_async_graph_path_parity(graph_sets, name):
    """medusa_materialize_async -> kernel_table_set -> restore(MEDUSA_N_SLOTS_FROM_TABLE),
    captured once into a CUDA graph and replayed (the bench's timed step), against the oracle."""
    gs = graph_sets(name)
    inp = medusa.upload(gs, DEV)
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size,
                             gs.func_id, gs.table)
    slots = medusa.alloc_slots(gs.n_words, DEV)
    res = torch.full((2,), -7, dtype=torch.int64, device=DEV)
    dst = torch.empty_like(inp["words"])
    fout = torch.empty(gs.n_nodes, dtype=torch.int64, device=DEV)
    rep = torch.empty(8, dtype=torch.int64, device=DEV)

    def step():
        medusa.materialize_async(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], out=slots, result=res)
        medusa.kernel_table_set(inp["table"])
        medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                       dst=dst, func_out=fout, report=rep, from_table=True)

    # eager async first (also sizes the library's scratch outside capture)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        step()
    torch.cuda.synchronize()
    assert medusa.mat_result(res) == (0, m["n_slots"])
    slots.n_slots = m["n_slots"]
    _check_materialize(slots, m, packed, gs.n_words)
    assert np.array_equal(medusa.to_numpy_u64(dst), packed[3])

    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    for _ in range(2):
        dst.zero_()
        fout.zero_()
        res.fill_(-7)
        slots.slot.fill_(-1)
        g.replay()
        torch.cuda.synchronize()
        assert medusa.mat_result(res) == (0, m["n_slots"])
        _check_materialize(slots, m, packed, gs.n_words)
        assert np.array_equal(medusa.to_numpy_u64(dst), packed[3])
        assert np.array_equal(medusa.to_numpy_u64(fout), packed[4])
        assert np.array_equal(medusa.report_numpy(rep), packed[5])


@pytest.mark.parametrize("name", ["toy", "llama2-13b"])
def test_stream_ordered_chain_without_host_sync(graph_sets, name):
    """In-place restore -> materialize_async of the restored image against the
    replayed trace -> kernel_table_set -> restore of that table, enqueued on one
    stream with no host synchronisation, five rounds: every programmatic launch
    (k_table_copy, k_zero, the early-triggering tail of each call) must order a
    read after the write it depends on.  Against the oracle run on the same chain."""
    gs = graph_sets(name)
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    m1, p1 = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size,
                          gs.func_id, gs.table)
    allocs2 = gs.allocs.copy()
    allocs2["base"] = gs.new_base  # the replayed trace: the restored image's pointers live here
    new_base2 = gs.new_base + np.uint64(1 << 36)
    table2 = gs.table.copy()
    table2[table2 != 0] += np.uint64(4096)
    m2, p2 = _oracle_full(p1[3], gs.node_word_off, gs.node_t, allocs2, new_base2, gs.new_size, gs.func_id, table2)
    assert m2["status"] == 0
    t64 = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int64)).to(DEV)  # noqa: E731
    allocs2_t = torch.from_numpy(np.ascontiguousarray(allocs2).view(np.int64).reshape(-1, 3)).to(DEV)
    nb2, tab2 = t64(new_base2), t64(table2)
    buf = torch.empty_like(inp["words"])
    dst2 = torch.empty_like(inp["words"])
    f1 = torch.empty(gs.n_nodes, dtype=torch.int64, device=DEV)
    f2 = torch.empty_like(f1)
    rep1 = torch.empty(8, dtype=torch.int64, device=DEV)
    rep2 = torch.empty_like(rep1)
    res = torch.empty(2, dtype=torch.int64, device=DEV)
    slots2 = medusa.alloc_slots(gs.n_words, DEV)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(5):
            buf.copy_(inp["words"])
            dst2.fill_(-1)
            medusa.kernel_table_set(inp["table"])
            medusa.restore(buf, slots, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"], dst=buf,
                           func_out=f1, report=rep1)
            medusa.materialize_async(buf, inp["node_off"], inp["node_t"], allocs2_t, out=slots2, result=res)
            medusa.kernel_table_set(tab2)
            medusa.restore(buf, slots2, inp["new_base"], nb2, inp["new_size"], inp["func_id"], dst=dst2, func_out=f2,
                           report=rep2, from_table=True)
    torch.cuda.synchronize()
    assert np.array_equal(medusa.to_numpy_u64(buf), p1[3])
    assert np.array_equal(medusa.to_numpy_u64(f1), p1[4])
    assert np.array_equal(medusa.report_numpy(rep1), p1[5])
    assert medusa.mat_result(res) == (0, m2["n_slots"])
    slots2.n_slots = m2["n_slots"]
    _check_materialize(slots2, m2, p2, gs.n_words)
    assert np.array_equal(medusa.to_numpy_u64(dst2), p2[3])
    assert np.array_equal(medusa.to_numpy_u64(f2), p2[4])
    assert np.array_equal(medusa.report_numpy(rep2), p2[5])


def test_async_reports_trace_error_and_capacity():
    """The async entry point reports what the synchronous one raises, in the result word."""
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(DEV)
    res = torch.zeros(2, dtype=torch.int64, device=DEV)
    seen_bad = seen_cap = False
    for seed in range(60):
        words, off, node_t, allocs = tiny_trace(seed * 11 + 3, overlap_p=0.2)
        o = oracle.materialize(words, off, node_t, allocs)
        aa = np.ascontiguousarray(allocs).view(np.int64).reshape(-1, 3) if allocs.size else np.zeros((0, 3), np.int64)
        inp = dict(words=t(words, np.int64), node_off=t(off, np.int64), node_t=t(node_t, np.int32),
                   allocs=torch.from_numpy(aa).to(DEV))
        medusa.materialize_async(**inp, out=medusa.alloc_slots(words.size, DEV), result=res)
        st, n = medusa.mat_result(res)
        assert st == o["status"], seed
        if st != 0:
            seen_bad = True
            continue
        assert n == o["n_slots"], seed
        if n > 0:
            medusa.materialize_async(**inp, out=medusa.alloc_slots(words.size, DEV, capacity=n - 1), result=res)
            assert medusa.mat_result(res) == (medusa.ERR_CAPACITY, n), seed
            seen_cap = True
    assert seen_bad and seen_cap


def _long_lived_mortals_trace(seed, n_mortal=1200, n_nodes=60000):
    """Many mortals live across the whole capture, one word per node: every chunk's
    window holds all of them (several batches), every chunk holds 2048 nodes (more
    than the node starts kept in shared memory), and the registration lists exceed
    the library's first guess (the overflow / exact-resize path)."""
    rng = np.random.default_rng(seed)
    base0 = 0x7F00_0000_0000
    t = 1
    allocs = []
    for i in range(n_mortal):  # disjoint, all live until the end of the capture
        allocs.append((base0 + i * 4096, 2048 if i % 7 else 0, t, 0))
        t += 1
    i_perm = []
    for k in range(16):  # a few I allocations (live at the last launch)
        allocs.append((base0 + (1 << 30) + k * 8192, 4096, t, T_NEVER))
        i_perm.append(len(allocs) - 1)
        t += 1
    node_t = []
    words = []
    for j in range(n_nodes):
        t += 1
        node_t.append(t)
        r = rng.random()
        if r < 0.5:
            a = allocs[int(rng.integers(0, n_mortal))]
            words.append(a[0] + int(rng.integers(0, 2049)))
        elif r < 0.7:
            a = allocs[i_perm[int(rng.integers(0, len(i_perm)))]]
            words.append(a[0] + int(rng.integers(0, 4097)))
        else:
            words.append(int(rng.integers(0, 1 << 62)))
    t += 1
    arr = np.zeros(len(allocs), ALLOC_DTYPE)
    for i, (b, sz, ta, tf) in enumerate(allocs):
        arr[i] = (b, sz, ta, tf if tf else t)  # mortals freed after the capture...
    t += 1
    node_t.append(t)  # ... and before one last launch, so they are not in I
    words.append(0)
    off = np.arange(len(words) + 1, dtype=np.uint64)
    return np.array(words, np.uint64), off, np.array(node_t, np.uint32), arr


@pytest.mark.parametrize("seed", [0, 1])
def test_overflow_retry_many_batches_wide_chunks(seed):
    words, off, node_t, allocs = _long_lived_mortals_trace(seed)
    m = oracle.materialize(words, off, node_t, allocs)
    assert m["status"] == 0
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(DEV)
    aa = np.ascontiguousarray(allocs).view(np.int64).reshape(-1, 3)
    inp = dict(words=t(words, np.int64), node_off=t(off, np.int64), node_t=t(node_t, np.int32),
               allocs=torch.from_numpy(aa).to(DEV))
    s = medusa.materialize(**inp)  # registrations overflow the first guess: resized, rerun
    mask, cb, rec = oracle.pack(m, words.size)
    assert s.n_slots == m["n_slots"]
    assert np.array_equal(_h(s.mask).view(np.uint32), mask)
    assert np.array_equal(_h(s.chunk_base).view(np.uint32), cb)
    assert np.array_equal(_h(s.slot[:s.n_slots]).view(np.uint64), rec)
    # the async entry now runs with the grown scratch
    res = torch.zeros(2, dtype=torch.int64, device=DEV)
    out = medusa.alloc_slots(words.size, DEV)
    medusa.materialize_async(**inp, out=out, result=res)
    assert medusa.mat_result(res) == (0, m["n_slots"])
    assert np.array_equal(_h(out.slot[:m["n_slots"]]).view(np.uint64), rec)


def test_malformed_csr_across_chunks_is_rejected_safely(graph_sets):
    """A non-monotone CSR spanning several chunks, and one whose last offset is not
    n_words, come back INVALID_ARG without touching memory out of range (the CUDA
    context stays usable: a valid ten-model call right after is bit-exact)."""
    b = 0x7F00_0000_0000
    w = np.uint64(b) + np.arange(4096, dtype=np.uint64) * np.uint64(8)
    A = np.array([(b, 8 * 4096, 1, T_NEVER)], dtype=ALLOC_DTYPE)
    nt = np.array([2, 3, 4], np.uint32)
    for off in ([0, 3000, 100, 4096], [0, 3000, 5000, 4096], [0, 100, 3000, 5000], [0, 2047, 6000, 9000],
                [7, 100, 2000, 4096]):
        st, _ = _run_tiny(w, np.array(off, np.uint64), nt, A)
        assert st == medusa.ERR_INVALID_ARG, off
    res = torch.zeros(2, dtype=torch.int64, device=DEV)
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(DEV)
    aa = torch.from_numpy(np.ascontiguousarray(A).view(np.int64).reshape(-1, 3)).to(DEV)
    medusa.materialize_async(t(w, np.int64), t(np.array([0, 3000, 100, 4096], np.uint64), np.int64),
                             t(nt, np.int32), aa, out=medusa.alloc_slots(w.size, DEV), result=res)
    assert medusa.mat_result(res)[0] == medusa.ERR_INVALID_ARG
    gs = graph_sets("all10")
    inp = medusa.upload(gs, DEV)
    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    m, packed = _oracle_full(gs.words, gs.node_word_off, gs.node_t, gs.allocs, gs.new_base, gs.new_size)
    _check_materialize(slots, m, packed, gs.n_words)
