"""NEXT-1 / NEXT-2 / NEXT-3 / NEXT-4 on the device: a real PyTorch decoder captured
into a CUDA graph, its allocation trace and kernel-node parameter image
materialized by libmedusa (checked against the oracle), restored for a second
address space (replayed allocations), written back into a clone of the
graph, and run: the output must equal the original graph's bit for bit, with
every original buffer poisoned."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU-only hosts
    pytest.skip("needs a GPU", allow_module_level=True)
pytest.importorskip("cuda.bindings.driver")

import oracle  # noqa: E402
from oracle import buffers as ob_  # noqa: E402
import paper_conf_asplos_zengxgcl25_b200 as medusa  # noqa: E402
from workloads.capture import real_graph  # noqa: E402


def test_real_graph_materialize_restore_replay():
    r = real_graph.end_to_end(torch, medusa)
    assert r["n_kernel"] > 20
    # allocations made during the capture exist (the graph's pool), and were
    # poisoned in the second arena before the rebuilt graph ran
    assert len(r["allocs"]) > r["n_pre"] > 0
    # the GPU table equals the oracle's on the real trace
    m = oracle.materialize(r["words"], r["off"], r["node_t"], r["allocs"])
    assert m["status"] == 0
    mask, cb, rec = oracle.pack(m, r["words"].size)
    s = r["slots"]
    assert s.n_slots == m["n_slots"] > 0
    assert np.array_equal(medusa.to_numpy_u64(s.slot[: s.n_slots]), rec)
    assert np.array_equal(s.mask.cpu().numpy().view(np.uint32), mask)
    # restore: every slot valid; the oracle restores the same bytes
    assert int(r["report"][0]) == 0
    dst_o, _, rep_o = oracle.restore(r["words"], m["slot_g"], m["slot_id"], m["slot_off"], r["allocs"]["base"],
                                     r["new_base"], r["allocs"]["size"])
    assert np.array_equal(r["restored"], dst_o) and int(rep_o[0]) == 0
    # copy-free buffer contents (§4.3): the plan equals the oracle's on the real
    # trace; the buffers holding the graphs' magic numbers are permanent
    cls = ob_.classify(r["allocs"], r["capture_t"], m["slot_id"])
    assert np.array_equal(r["buf_class"], cls)
    perm, poff = ob_.plan(r["allocs"], cls)
    assert np.array_equal(r["perm"], perm) and np.array_equal(r["perm_off"].view(np.uint64), poff)
    assert r["n_perm"] >= 1 and all(cls[i] == ob_.PERM for i in r["magic_allocs"])
    assert (cls == ob_.PARAM).sum() > 0  # weights, inputs, mask: allocated before capturing
    assert r["buf_report"] == [0, 2**64 - 1, 0, 2**64 - 1]
    # every rebuilt graph computes the same output, bit for bit -- and without the
    # permanent buffers' contents it does not
    assert r["n_graphs"] == 4
    for ob, ref in zip(r["outs_b"], r["refs"]):
        assert torch.equal(ob, ref)
    assert not any(torch.equal(ob, ref) for ob, ref in zip(r["outs_unrestored"], r["refs"]))


def test_fresh_process_online_phase(tmp_path):
    """Offline and online phases in two fresh processes: same loading sequence,
    replayed allocations, kernel addresses by dlsym + first-layer triggering
    capture + module enumeration (§5), restore with the kernel-address fill,
    every graph built from scratch (cuGraphAddKernelNode): outputs bit-identical."""
    import json
    import os
    import subprocess
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    tool = os.path.join(root, "tools", "real_capture_online.py")

    def phase(name):  # each phase in a process of its own (fresh CUDA state)
        r = subprocess.run([sys.executable, tool, name, str(tmp_path)], capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-2000:]
        return json.loads(r.stdout.strip().splitlines()[-1])

    off = phase("offline")
    assert off["names"] > 10 and off["slots"] > 0 and off["n_perm"] >= 1
    res = phase("online")
    assert res["same_loading"]
    assert res["kernels"]["unresolved"] == 0
    assert res["report"][0] == 0 and res["report"][5] == 0  # no bad slot, no unresolved kernel
    assert res["moved_bases"] == res["allocations"]  # a genuinely different address space
    assert res["buf_report"] == [0, 2**64 - 1]  # every permanent buffer's contents restored (§4.3)
    assert res["outputs_equal"] and all(res["outputs_equal"])
