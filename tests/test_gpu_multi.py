"""Every visible GPU restores its own C5 instance concurrently (SURVEY.md §8(e):
one Llama-2-13B-shaped instance per GPU, seed 100 + gpu, no collective), one
host thread per instance; each GPU's table, restored words, kernel addresses and
report are compared with the oracle.  A second instance shares each device as
well (its own thread and stream: the per-device materialize lock serializes the
two without blocking other devices).  The kernel-address table is per device,
so only the first instance of a device runs the kernel-address fill."""
import threading

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU-only hosts
    pytest.skip("needs a GPU", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_asplos_zengxgcl25_b200 as medusa  # noqa: E402
from workloads import make_graph_set  # noqa: E402


def _expected(gs, gather):
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    mask, cb, rec = oracle.pack(m, gs.n_words)
    dst, fout, rep = oracle.restore(gs.words, m["slot_g"], m["slot_id"], m["slot_off"], gs.allocs["base"],
                                    gs.new_base, gs.new_size, gs.func_id if gather else None,
                                    gs.table if gather else None)
    return m["n_slots"], mask, cb, rec, dst, fout, rep


def test_every_gpu_restores_its_own_instance_concurrently():
    n_dev = torch.cuda.device_count()
    # (device, seed, gather): instance g = seed 100 + g; the first n_dev ones one per device
    jobs = [(g % n_dev, 100 + g, g < n_dev) for g in range(2 * n_dev)]
    sets = {seed: make_graph_set("llama2-13b", seed=seed) for _, seed, _ in jobs}
    out, errs = {}, []
    start = threading.Barrier(len(jobs))

    def run(dev_i, seed, gather):
        try:
            dev = torch.device("cuda", dev_i)
            torch.cuda.set_device(dev)
            gs = sets[seed]
            s = torch.cuda.Stream(dev)
            with torch.cuda.stream(s):
                inp = medusa.upload(gs, dev)
                s.synchronize()
                start.wait()
                for _ in range(3):  # several rounds, so the threads' calls interleave
                    slots = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], stream=s)
                    if gather:
                        medusa.kernel_table_set(inp["table"], stream=s)
                    dst, fout, rep = medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"],
                                                    inp["new_size"], inp["func_id"] if gather else None, stream=s)
                s.synchronize()
                h = lambda t: t.detach().cpu().numpy()
                out[seed] = (slots.n_slots, h(slots.mask).view(np.uint32), h(slots.chunk_base).view(np.uint32),
                             h(slots.slot[:slots.n_slots]).view(np.uint64), medusa.to_numpy_u64(dst),
                             medusa.to_numpy_u64(fout) if gather else None, medusa.report_numpy(rep))
        except Exception as e:  # pragma: no cover - reported below
            errs.append((seed, repr(e)))

    th = [threading.Thread(target=run, args=j) for j in jobs]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert not errs, errs
    for _, seed, gather in jobs:
        got, exp = out[seed], _expected(sets[seed], gather)
        assert got[0] == exp[0], seed
        for k in (1, 2, 3, 4, 6):
            assert np.array_equal(got[k], exp[k]), (seed, k)
        if gather:
            assert np.array_equal(got[5], exp[5]), seed
    assert len({out[s][0] for _, s, _ in jobs}) > 1  # the instances differ
