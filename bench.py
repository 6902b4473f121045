"""Benchmark of the Medusa restoration hot path on B200 (one JSON line on rank 0).

A step = one pass of the whole hot path over one graph set already resident in
HBM: medusa_kernel_table_set (install the triggering-kernel address table;
independent of the analysis) -> medusa_materialize (classify every word + emit
the indirect-index-pointer table) -> medusa_restore (relocate + validate every
slot, fill every node's kernel address).  Metric (BASELINE.json): graph nodes
restored per second, whole job; plus the relocate pass's HBM GB/s.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload all10] [--impl ours|reference]

Multi-GPU: the path shards per instance, so every rank (one
process per GPU) restores its own independently generated instance and no data
crosses GPUs.  `--gpus N` without WORLD_SIZE in the environment starts the N
rank processes itself; under torchrun WORLD_SIZE must equal N.  The ranks meet
only on the host: a gloo process group supplies the start/stop barriers, the
max over ranks of the device-timed regions and the gathering of per-rank
results -- no NCCL, no collective on the data path.  Every rank runs
  * the headline workload (`--workload`, default the ten-model set; rank r's
    instance is generated with seed + 1000 r): value = N x nodes x K / max_r t_r;
  * C5 (BASELINE.json configs[4]): its own Llama-2-13B-shaped instance with seed
    100 + r, timed concurrently on every GPU: aggregate nodes/s
    = sum of nodes / max time, per-GPU relocate GB/s, sustained relocate per GPU;
  * parity: after timing, each rank's table, restored words, kernel addresses
    and report of both workloads are compared with the CPU oracle.
--impl reference times the CPU oracle (oracle/, plain C++) on the same config.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    "all10": ("all10", "ten paper models concatenated (Table 1: 139,364 nodes), one call"),
    "qwen1.5-4b": ("qwen1.5-4b", "Qwen1.5-4B-shaped graph set, 35 batch sizes (16,150 nodes)"),
    "llama2-7b": ("llama2-7b", "Llama-2-7B-shaped graph set with kernel table (12,518 nodes)"),
    "llama2-13b": ("llama2-13b", "Llama-2-13B-shaped instance (16,150 nodes)"),
    "toy": ("toy", "toy 2-layer decoder, 200 nodes"),
    "all10-inband": ("all10-inband", "stress: the ten-model set with ~8% of words in-band non-pointer constants "
                                     "(VA holes, freed memory)"),
}
# the paper's own end-to-end numbers, quoted beside ours: another
# machine's, not the target (the paper never times these passes on their own)
PAPER_CONTEXT = {
    "hardware": "1 x NVIDIA A100-40GB SXM4, 2 x AMD EPYC 7642, PyTorch 2.2.0, CUDA 12.4 (P:271, P:405-415)",
    "online_capture_stage_s": {"value": 0.57, "vllm": 0.90, "workload": "Qwen1.5-4B, 16,150 nodes, 35 batch sizes",
                               "cite": "P:311-319", "implied_restore_rate_lower_bound_nodes_per_s": 28300},
    "offline_phase_s_per_model": {"value": 39.2, "capture_s": 9.7, "implied_analysis_nodes_per_s": 472,
                                  "cite": "P:325"},
    "loading_phase_reduction_vs_vllm": 0.425, "cold_start_reduction_avg": 0.349, "p99_ttft_reduction": 0.530,
    "cite_reductions": "P:44, P:287-291, P:329-343",
}
SEED_STRIDE = 1000  # rank r restores the instance generated with seed + r * SEED_STRIDE


def path_counts(gs, slot_id=None):
    """Host-side counts the per-kernel algorithmic bytes need (from the inputs and,
    for the window / I-list split, the oracle's slot ids when given)."""
    a = gs.allocs
    nt = gs.node_t
    t_last = int(nt[-1]) if nt.size else 0
    live = a["size"] > 0
    isI = live & (a["t_alloc"] < t_last) & (t_last < a["t_free"]) if nt.size else np.zeros(a.size, bool)
    gmin = int(a["base"][live].min()) if live.any() else 0
    gmax = int((a["base"][live] + a["size"][live]).max()) if live.any() else 0
    w = gs.words
    cand = int(((w >= np.uint64(gmin)) & (w < np.uint64(gmax))).sum()) if gmax else 0
    n_i = int(isI.sum())
    out = {"n_I": n_i, "candidates": cand}
    if slot_id is not None:
        i_hits = int(isI[slot_id.astype(np.int64)].sum())
        out.update(i_hits=i_hits, window_hits=int(slot_id.size) - i_hits, queued=cand - (int(slot_id.size) - i_hits))
    return out


def algorithmic_bytes(gs, n_slots, n_func, counts=None):
    """Bytes the method itself must move per launch of each kernel (SURVEY.md
    §8(d) for mat_classify = K1+K2 and restore = K3+K4; DESIGN.md §5 for the
    others: what the kernel must read and write, intermediate structures included,
    at their per-unit sizes)."""
    W, N, A = gs.n_words, gs.n_nodes, gs.n_alloc
    n_mask = (W + 31) // 32
    C = (W + 2047) // 2048
    restore = (16 * W + 4 * n_mask + 4 * (C + 1) + 8 * n_slots + 24 * A + 12 * N + 8 * n_func + 64)
    classify = (8 * W + 4 * n_mask + 4 * (C + 1) + 8 * n_slots + 12 * N)
    # in place (dst == src): only the slot words are read and written
    inplace = (4 * n_mask + 4 * (C + 1) + 8 * n_slots + 16 * n_slots + 24 * A + 12 * N + 8 * n_func + 64)
    out = dict(restore=restore, mat_classify=classify, restore_inplace=inplace)
    if counts is not None and "queued" in counts:
        nI, q = counts["n_I"], counts["queued"]
        T = max(1, (nI + 1023) // 1024)
        out.update(
            # records + node CSR in; tree leaves (8 B/alloc), tree nodes, I keys (12 B), chunk node ranges (16 B)
            mat_trace=24 * A + 12 * N + 8 * A + 8 * ((A + 31) // 32) + 12 * nI + 16 * C,
            mat_isort=24 * nI,                                     # I keys in, sorted tiles out
            # each key + per other tile one 32-key sample block and one 32-key block (12 B/key), I entry out
            mat_rank=(12 * nI + 24 * (T - 1) * nI + 52 * nI) if T > 1 else 0,
            mat_iresolve=16 * q + 8 * counts["i_hits"] + 8 * n_mask,   # queue in, records + masks out
            mat_emit=3 * 4 * n_mask + 16 * n_slots + 4 * (C + 1),    # 3 masks, records in + table out
            mat_check_mm=24 * A + 8 * A,                          # own records, tree leaves
            mat_check_mi=24 * A + 28 * nI,                        # own records, the sorted I list
            restore_report_init=64,
        )
    return out


def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def load_traffic(workload):
    """Per-launch DRAM bytes (and warp instructions, `_inst`) of each kernel of this
    workload, from the committed ncu launch list of the same command
    (profiles/ncu_traffic.json, one entry per workload); {} if none was captured
    for it (then `traffic` is null: another workload's counters are never used)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        return json.load(open(p)).get(workload, {})
    except Exception:
        return {}


class ClockSampler:
    """SM clock and throttle reasons sampled DURING the timed region: after the
    K steps are enqueued, the host polls NVML until the last step's end event
    has fired (nvidia-smi's 50 ms loop cannot land inside a ~6 ms region)."""
    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4), ("hw_power_brake_slowdown", 0x80))

    def __init__(self, gpu_index):
        self.rows, self.h, self.max_mhz = [], None, 0.0
        try:
            import pynvml
            pynvml.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            parts = vis.split(",") if vis else []
            idx = int(parts[gpu_index]) if gpu_index < len(parts) and parts[gpu_index].isdigit() else gpu_index
            self.h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self.nvml = pynvml
            self.max_mhz = float(pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM))
        except Exception:
            self.h = None

    def sample(self):
        if self.h is None:
            return
        try:
            sm = self.nvml.nvmlDeviceGetClockInfo(self.h, self.nvml.NVML_CLOCK_SM)
            rs = self.nvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            self.rows.append((float(sm), int(rs)))
        except Exception:
            pass

    def poll_until(self, event):
        """Samples while the GPU is still inside the timed region (event not yet reached)."""
        while not event.query():
            self.sample()

    def stop(self):
        rows = self.rows
        if not rows:
            return None
        loaded = [r for r in rows if r[0] > 0.5 * self.max_mhz] or rows
        reasons = sorted({nm for r in rows for nm, bit in self.REASONS if r[1] & bit})
        return {"sm_mhz": statistics.median(r[0] for r in loaded), "sm_max_mhz": self.max_mhz, "reasons": reasons,
                "samples": len(rows), "samples_under_load": len(loaded),
                "source": "NVML, polled by the host between enqueueing the K timed steps and the last step's end event"}


def graph_kernel_nodes(graph):
    """Kernel nodes of a captured torch CUDA graph (driver API: cuGraphGetNodes /
    cuGraphNodeGetType; CU_GRAPH_NODE_TYPE_KERNEL = 0)."""
    import ctypes
    cu = ctypes.CDLL("libcuda.so.1")
    g = ctypes.c_void_p(graph.raw_cuda_graph())
    n = ctypes.c_size_t(0)
    assert cu.cuGraphGetNodes(g, None, ctypes.byref(n)) == 0
    nodes = (ctypes.c_void_p * n.value)()
    assert cu.cuGraphGetNodes(g, nodes, ctypes.byref(n)) == 0
    k, t = 0, ctypes.c_int()
    for i in range(n.value):
        assert cu.cuGraphNodeGetType(ctypes.c_void_p(nodes[i]), ctypes.byref(t)) == 0
        k += t.value == 0
    return k


C5 = "llama2-13b"  # BASELINE.json configs[4]: one Llama-2-13B-shaped instance per GPU, seed 100 + gpu


def rank_seed(cfg, rank):
    """Seed of the independent instance rank `rank` restores (weak scaling):
    C5 uses 100 + rank, the other configs seed + 1000 rank."""
    from workloads.graphset import CONFIGS
    if cfg == C5:
        return CONFIGS[cfg]["seed"] + rank
    return CONFIGS[cfg]["seed"] + SEED_STRIDE * rank


def max_over_ranks(x, dist, device=None):
    """Max of a per-rank scalar over all ranks (the job's time is the slowest rank's),
    over the host-side gloo group (no device collective)."""
    import torch
    t = torch.tensor([float(x)], dtype=torch.float64)
    if dist is not None and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_to_all(obj, dist):
    """Every rank's `obj`, in rank order (gloo all_gather_object; [obj] on one rank)."""
    if dist is not None and dist.is_initialized() and dist.get_world_size() > 1:
        out = [None] * dist.get_world_size()
        dist.all_gather_object(out, obj)
        return out
    return [obj]


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    return int(os.environ.get("RANK", "0")), ws, int(os.environ.get("LOCAL_RANK", "0"))


def config_dict(cfg, desc, gs, n_slots, seed, ws):
    """The `config` object of the JSON line -- identical for both arms."""
    return {"workload": f"{cfg} per rank: {desc}", "nodes_per_rank": gs.n_nodes, "words": gs.n_words,
            "allocs": gs.n_alloc, "slots": int(n_slots), "kernel_names": int(gs.table.size), "seed": seed,
            "l2": "GPU arm: 256 MiB (2x L2) scrub written before every timed step; CPU arm: not applicable",
            "parallelism": f"{ws} independent instances (one per GPU), no collective"}


def plumbing_selftest(args):
    """`--selftest-plumbing` (CPU, tests/test_multi.py): the multi-rank plumbing of
    run_ours without a GPU -- the gloo group the launcher's env describes, a
    barrier, the max of a rank-dependent time, the gather -- printed by rank 0.
    Produces no bench value."""
    import torch.distributed as dist
    rank, ws, local = dist_env()
    if ws > 1:
        dist.init_process_group("gloo", rank=rank, world_size=ws)
        dist.barrier()
    t = max_over_ranks(10.0 + rank, dist)
    got = gather_to_all({"rank": rank, "local": local, "seed_c5": rank_seed(C5, rank),
                         "seed_all10": rank_seed("all10", rank), "pid": os.getpid()}, dist)
    if rank == 0:
        print(json.dumps({"world_size": ws, "max_ms": t, "ranks": got}), flush=True)
    if ws > 1:
        dist.barrier()
        dist.destroy_process_group()


def spawn_ranks(args, n_visible=None):
    """`--gpus N` outside torchrun: start N rank processes of this script (RANK /
    LOCAL_RANK / WORLD_SIZE / MASTER_* set as torchrun would) and wait for them."""
    import socket
    import subprocess
    if n_visible is None:
        import torch
        n_visible = torch.cuda.device_count()
    n_dev = n_visible
    if n_dev < args.gpus:
        raise SystemExit(f"bench.py --gpus {args.gpus}: only {n_dev} GPU(s) visible")
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    procs = []
    for r in range(args.gpus):
        env = dict(os.environ, RANK=str(r), LOCAL_RANK=str(r), WORLD_SIZE=str(args.gpus),
                   LOCAL_WORLD_SIZE=str(args.gpus), MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        procs.append(subprocess.Popen([sys.executable, os.path.abspath(__file__), *sys.argv[1:]], env=env))
    rcs = [p.wait() for p in procs]
    if any(rcs):
        raise SystemExit(f"bench.py rank exit codes {rcs}")


def run_reference(args):
    """--impl reference: the CPU oracle, as it stands, on this arm's config."""
    rank, ws, _ = dist_env()
    if rank != 0:
        return
    import __graft_entry__ as ge
    ge.build_oracle()
    import oracle
    from workloads import make_graph_set

    cfg, desc = WORKLOADS[args.workload]
    seed = rank_seed(cfg, 0)
    gs = make_graph_set(cfg, seed=seed)
    n_slots = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)["n_slots"]

    def step():
        m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
        oracle.restore(gs.words, m["slot_g"], m["slot_id"], m["slot_off"], gs.allocs["base"], gs.new_base,
                       gs.new_size, gs.func_id, gs.table)

    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    dt = time.perf_counter() - t0
    value = gs.n_nodes * args.steps / dt
    print(json.dumps({
        "impl": "reference", "metric": "graph nodes restored/sec (materialize + restore, whole hot path)",
        "value": value, "unit": "nodes/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * dt / args.steps, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "u64", "data": "synthetic",
        "config": config_dict(cfg, desc, gs, n_slots, seed, args.gpus),
        "cpu_baseline": {"value": value, "unit": "nodes/s", "cores": 1, "kind": "oracle",
                         "sample": f"full {cfg} graph set per step (materialize + restore), single-threaded "
                                   f"oracle/oracle.cpp (-O2), on rank 0 only"},
        "e2e": {"value": value, "unit": "nodes/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_all_cores(oracle, gs, seconds):
    """SURVEY.md §8(d) oracle timing (b): the unchanged oracle on every host core.
    The node range is split into one contiguous part per thread for MATERIALIZE
    (each part is a complete sub-problem: a word's class depends only on its node's
    launch position and the whole trace, which every part receives) and the word
    range for RESTORE (each part gets its slots, rebased; the kernel-address
    gather runs with the first part).  Python threads around ctypes calls (the GIL
    is released inside the oracle).  Returns (nodes/s, materialize nodes/s,
    restore nodes/s, threads, passes); the parts' outputs are checked against the
    single-threaded run on the first pass."""
    import threading
    P = os.cpu_count() or 1
    N, W = gs.n_nodes, gs.n_words
    off = gs.node_word_off.astype(np.int64)
    jcut = [N * k // P for k in range(P + 1)]
    wcut = [int(off[j]) for j in jcut]

    def run_parallel(fn):
        out = [None] * P
        th = [threading.Thread(target=lambda k=k: out.__setitem__(k, fn(k))) for k in range(P)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        return out

    def mat_part(k):
        j0, j1 = jcut[k], jcut[k + 1]
        w0, w1 = wcut[k], wcut[k + 1]
        m = oracle.materialize(gs.words[w0:w1], (off[j0:j1 + 1] - w0).astype(np.uint64), gs.node_t[j0:j1], gs.allocs)
        return m["slot_g"] + np.uint64(w0), m["slot_id"], m["slot_off"]

    ref = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    ref_dst = oracle.restore(gs.words, ref["slot_g"], ref["slot_id"], ref["slot_off"], gs.allocs["base"],
                             gs.new_base, gs.new_size, gs.func_id, gs.table)[0]
    t_mat = t_res = 0.0
    reps = 0
    t_start = time.perf_counter()
    while time.perf_counter() - t_start < seconds or reps == 0:
        t1 = time.perf_counter()
        parts = run_parallel(mat_part)
        t2 = time.perf_counter()
        g = np.concatenate([q[0] for q in parts])
        sid = np.concatenate([q[1] for q in parts])
        soff = np.concatenate([q[2] for q in parts])
        bounds = np.searchsorted(g, np.array(wcut, dtype=np.uint64))
        dst = np.empty_like(gs.words)

        def res_part(k):
            w0, w1 = wcut[k], wcut[k + 1]
            s0, s1 = bounds[k], bounds[k + 1]
            first = k == 0
            d, _, _ = oracle.restore(gs.words[w0:w1], g[s0:s1] - np.uint64(w0), sid[s0:s1], soff[s0:s1],
                                     gs.allocs["base"], gs.new_base, gs.new_size,
                                     gs.func_id if first else None, gs.table if first else None)
            dst[w0:w1] = d

        t3 = time.perf_counter()
        run_parallel(res_part)
        t4 = time.perf_counter()
        if reps == 0:
            assert np.array_equal(g, ref["slot_g"]) and np.array_equal(soff, ref["slot_off"])
            assert np.array_equal(dst, ref_dst)
        t_mat += t2 - t1
        t_res += t4 - t3
        reps += 1
    return N * reps / (t_mat + t_res), N * reps / t_mat, N * reps / t_res, P, reps


def bench_inplace(medusa, gs, inp, slots, dev, stream, scrub, steps, peak, alg, replicas):
    import torch
    from workloads.graphset import replicate

    def run(x, xin, sl, reps, scrub_each):
        buf = xin["words"].clone()
        fout = torch.empty(x.n_nodes, dtype=torch.int64, device=dev)
        rep = torch.empty(8, dtype=torch.int64, device=dev)
        fwd = (xin["old_base"], xin["new_base"])
        medusa.kernel_table_set(xin["table"])

        def call(k):
            ob, nb = fwd if k % 2 == 0 else fwd[::-1]
            medusa.restore(buf, sl, ob, nb, xin["new_size"], xin["func_id"], dst=buf, func_out=fout, report=rep)
        for k in range(4):
            call(k)
        torch.cuda.synchronize(dev)
        assert int(medusa.report_numpy(rep)[0]) == 0 and torch.equal(buf, xin["words"])
        medusa.timing_enable(True)
        for k in range(reps):
            if scrub_each:
                scrub.fill_(k)
            call(k)
        ts = [ms for name, ms in medusa.timing_read(1 << 16) if name == "restore"]
        medusa.timing_enable(False)
        torch.cuda.synchronize(dev)
        assert int(medusa.report_numpy(rep)[0]) == 0
        a = algorithmic_bytes(x, sl.n_slots, x.table.size)["restore_inplace"]
        t = statistics.median(ts) / 1e3
        return {"avg_us": t * 1e6, "alg_bytes": a, "GB/s": a / t / 1e9, "frac_of_peak": a / t / 1e9 / peak,
                "nodes_per_s": x.n_nodes / t}

    out = {"all10": run(gs, inp, slots, steps, True)}
    if replicas > 0:
        big = replicate(gs, replicas)
        binp = medusa.upload(big, dev)
        bsl = medusa.materialize(binp["words"], binp["node_off"], binp["node_t"], binp["allocs"])
        out[f"x{replicas}"] = run(big, binp, bsl, 10, False)
        del binp, bsl, big
        torch.cuda.empty_cache()
    medusa.kernel_table_set(inp["table"])
    out["note"] = ("medusa_restore with dst == src: per slot the record, 24 B of replay table and the 8-B word "
                   "read + written; the other words are not touched; kernel-only time (per-launch events), median")
    return out


def bench_buffers(medusa, gs, inp, slots, dev, stream, scrub, steps, peak):
    """medusa_buffers_plan (offline, synchronous) and medusa_buffers_save /
    medusa_buffers_restore (offline dump / online copy-back) on the workload.  The
    synthetic trace's addresses are not device memory, so the permanent buffers get
    real ones: an arena in ordinal order (old) and one in shuffled order (new)."""
    import torch
    ev = lambda: torch.cuda.Event(enable_timing=True)
    plan = medusa.buffers_plan(inp["allocs"], inp["capture_t"], slots.slot, slots.n_slots)
    torch.cuda.synchronize(dev)
    perm = plan.perm.cpu().numpy().view(np.uint32)
    sizes = gs.allocs["size"][perm].astype(np.int64)
    old_arena = torch.randint(0, 256, (max(int(sizes.sum()), 16),), dtype=torch.uint8, device=dev)
    new_arena = torch.zeros_like(old_arena)
    pos = np.concatenate([[0], np.cumsum(sizes)[:-1]]).astype(np.int64)
    base = np.zeros(gs.n_alloc, np.uint64)
    nb = np.zeros(gs.n_alloc, np.uint64)
    base[perm] = old_arena.data_ptr() + pos
    nb[perm[np.random.default_rng(0).permutation(perm.size)]] = new_arena.data_ptr() + pos
    d_base = torch.from_numpy(base.view(np.int64)).to(dev)
    d_nb = torch.from_numpy(nb.view(np.int64)).to(dev)
    blob = torch.empty(max(plan.blob_bytes, 16), dtype=torch.uint8, device=dev)
    rep = torch.empty(2, dtype=torch.int64, device=dev)
    for _ in range(3):
        medusa.buffers_plan(inp["allocs"], inp["capture_t"], slots.slot, slots.n_slots)
        medusa.buffers_save(plan, d_base, blob=blob, report=rep)
        medusa.buffers_restore(plan, blob, d_nb, inp["new_size"], report=rep)
    torch.cuda.synchronize(dev)
    assert torch.equal(blob[:plan.blob_bytes], old_arena[:plan.blob_bytes])
    assert int(rep[0].item()) == 0

    def t(fn):
        out = []
        for k in range(steps):
            scrub.fill_(k)
            a, b = ev(), ev()
            a.record(stream)
            fn()
            b.record(stream)
            out.append((a, b))
        torch.cuda.synchronize(dev)
        return statistics.median(a.elapsed_time(b) for a, b in out)

    plan_ms = t(lambda: medusa.buffers_plan(inp["allocs"], inp["capture_t"], slots.slot, slots.n_slots))
    # save / restore are asynchronous and capturable: each one captured into a CUDA
    # graph and replayed, so the events see device time, not Python launch gaps
    graphs = {}
    for name, fn in (("save", lambda: medusa.buffers_save(plan, d_base, blob=blob, report=rep)),
                     ("restore", lambda: medusa.buffers_restore(plan, blob, d_nb, inp["new_size"], report=rep))):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            fn()
        graphs[name] = g
    save_ms = t(graphs["save"].replay)
    rest_ms = t(graphs["restore"].replay)
    torch.cuda.synchronize(dev)
    ok = int(rep[0].item()) == 0 and torch.equal(new_arena[:plan.blob_bytes].sort().values,
                                                 old_arena[:plan.blob_bytes].sort().values)
    # kernel-only durations (libmedusa's per-launch events around each launch; these
    # include the host's launch latency when the GPU is idle), L2 scrubbed before each call
    medusa.timing_enable(True)
    for k in range(steps):
        scrub.fill_(k)
        medusa.buffers_save(plan, d_base, blob=blob, report=rep)
        scrub.fill_(k)
        medusa.buffers_restore(plan, blob, d_nb, inp["new_size"], report=rep)
    kt = {}
    for name, ms in medusa.timing_read(1 << 16):
        kt.setdefault(name, []).append(ms)
    medusa.timing_enable(False)
    kernel_us = {n: 1e3 * statistics.median(v) for n, v in kt.items()}
    moved = 2 * plan.blob_bytes + 12 * plan.n_perm + 8 * plan.n_perm  # bytes + perm/off + base(+size)
    return {"n_perm": plan.n_perm, "perm_kernel_frac": float(gs.node_perm.mean()), "blob_bytes": plan.blob_bytes,
            "classes": {k: int((plan.cls == v).sum().item()) for k, v in
                        (("unused", 0), ("param", 1), ("temp", 2), ("perm", 3))},
            "plan_ms": plan_ms, "save_us": save_ms * 1e3, "restore_us": rest_ms * 1e3,
            "restore_GB/s": moved / (rest_ms / 1e3) / 1e9, "restore_frac_of_peak": moved / (rest_ms / 1e3) / 1e9 / peak,
            "restore_ok": ok, "kernel_us": kernel_us,
            "restore_events_GB/s": moved / (kernel_us["buf_restore"] / 1e6) / 1e9,
            "note": "save_us / restore_us: median of K graph replays of one call (device time incl. the graph "
                    "launch), L2 scrubbed before each; medusa_buffers_restore = the online copy-back (P:220-224), "
                    "bytes = 2 x blob + 20 B per buffer"}


def oracle_parity(gs, slots, n_slots, dst, fout, rep):
    """This rank's GPU outputs against the CPU oracle on the same instance: the
    table (mask, chunk prefix, records), restored words, kernel addresses, report."""
    import oracle
    import paper_conf_asplos_zengxgcl25_b200 as medusa
    m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
    if m["status"] != 0:
        return {"ok": False, "why": f"oracle status {m['status']}"}
    mask, cb, rec = oracle.pack(m, gs.n_words)
    odst, ofout, orep = oracle.restore(gs.words, m["slot_g"], m["slot_id"], m["slot_off"], gs.allocs["base"],
                                       gs.new_base, gs.new_size, gs.func_id, gs.table)
    h = lambda t: t.detach().cpu().numpy()
    checks = {
        "n_slots": n_slots == m["n_slots"],
        "mask": np.array_equal(h(slots.mask).view(np.uint32), mask),
        "chunk_base": np.array_equal(h(slots.chunk_base).view(np.uint32), cb),
        "records": np.array_equal(h(slots.slot[:m["n_slots"]]).view(np.uint64), rec),
        "words": np.array_equal(medusa.to_numpy_u64(dst), odst),
        "func_out": np.array_equal(medusa.to_numpy_u64(fout), ofout),
        "report": np.array_equal(medusa.report_numpy(rep), orep),
    }
    return {"ok": all(checks.values()), "failed": [k for k, v in checks.items() if not v],
            "slots": int(m["n_slots"]), "words": gs.n_words}, m["slot_id"]


def bench_c5(medusa, args, rank, dev, stream, scrub, barrier, peak):
    """C5 (BASELINE.json configs[4]): this rank's own
    Llama-2-13B-shaped instance (seed 100 + rank), the whole-path step captured
    as one CUDA graph and timed on every GPU at once (barrier-bracketed device
    events); the restore alone (latency mode, graph replays); one sustained
    restore over R replicas; parity with the oracle after timing."""
    import torch
    from workloads import make_graph_set
    from workloads.graphset import replicate
    seed = rank_seed(C5, rank)
    gs = make_graph_set(C5, seed=seed)
    inp = medusa.upload(gs, dev)
    sl = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])  # sizes the scratch
    n_slots = sl.n_slots
    res = torch.zeros(2, dtype=torch.int64, device=dev)
    dst = torch.empty_like(inp["words"])
    fout = torch.empty(gs.n_nodes, dtype=torch.int64, device=dev)
    rep = torch.empty(8, dtype=torch.int64, device=dev)
    medusa.kernel_table_set(inp["table"])

    def step():
        medusa.kernel_table_set(inp["table"])
        medusa.materialize_async(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], out=sl, result=res)
        medusa.restore(inp["words"], sl, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                       dst=dst, func_out=fout, report=rep, from_table=True)

    def rest():
        medusa.restore(inp["words"], sl, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                       dst=dst, func_out=fout, report=rep, from_table=True)

    graphs = {}
    for name, fn in (("step", step), ("restore", rest)):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            fn()
        graphs[name] = g
    for _ in range(3):
        graphs["step"].replay()
    torch.cuda.synchronize(dev)

    def timed(g):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        barrier()
        for k in range(args.steps):
            scrub.fill_(k)
            ev[k][0].record(stream)
            g.replay()
            ev[k][1].record(stream)
        barrier()
        return [a.elapsed_time(b) for a, b in ev]

    step_ms = timed(graphs["step"])
    rest_ms = timed(graphs["restore"])
    st, ns = medusa.mat_result(res)
    assert st == 0 and ns == n_slots, (st, ns)
    par = oracle_parity(gs, sl, n_slots, dst, fout, rep)[0]
    alg = algorithmic_bytes(gs, n_slots, gs.table.size)["restore"]
    t_rest = statistics.median(rest_ms) / 1e3
    out = {"rank": rank, "seed": seed, "nodes": gs.n_nodes, "words": gs.n_words, "slots": n_slots,
           "sum_ms": sum(step_ms), "ms_per_step": statistics.median(step_ms),
           "relocate_us": t_rest * 1e6, "relocate_GB/s": alg / t_rest / 1e9, "relocate_frac": alg / t_rest / 1e9 / peak,
           "parity": par}
    del graphs
    if args.c5_sustained > 0:
        R = args.c5_sustained
        big = replicate(gs, R)
        binp = medusa.upload(big, dev)
        bsl = medusa.materialize(binp["words"], binp["node_off"], binp["node_t"], binp["allocs"])
        medusa.kernel_table_set(binp["table"])
        bdst = torch.empty_like(binp["words"])
        bfout = torch.empty(big.n_nodes, dtype=torch.int64, device=dev)
        brep = torch.empty(8, dtype=torch.int64, device=dev)
        call = lambda: medusa.restore(binp["words"], bsl, binp["old_base"], binp["new_base"], binp["new_size"],
                                      binp["func_id"], dst=bdst, func_out=bfout, report=brep)
        for _ in range(2):
            call()
        torch.cuda.synchronize(dev)
        assert int(medusa.report_numpy(brep)[0]) == 0
        balg = algorithmic_bytes(big, bsl.n_slots, big.table.size)["restore"]
        reps = 10
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        e0.record(stream)
        for _ in range(reps):
            call()
        e1.record(stream)
        barrier()
        t = e0.elapsed_time(e1) / 1e3 / reps
        out["sustained"] = {"replicas": R, "alg_bytes": balg, "avg_ms": t * 1e3, "GB/s": balg / t / 1e9,
                            "frac_of_peak": balg / t / 1e9 / peak, "nodes_per_s": big.n_nodes / t}
        medusa.kernel_table_set(inp["table"])
        del binp, bsl, bdst, bfout, big
        torch.cuda.empty_cache()
    return out


def run_ours(args):
    import torch
    import torch.distributed as dist

    import __graft_entry__ as ge
    ge.build_medusa()
    import paper_conf_asplos_zengxgcl25_b200 as medusa
    from workloads import make_graph_set
    rank, ws, local = dist_env()
    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a GPU (there is no CPU fallback)")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if ws > 1:  # host-side group only: barriers, max of device times, per-rank results (no NCCL)
        dist.init_process_group("gloo", rank=rank, world_size=ws)

    cfg, desc = WORKLOADS[args.workload]
    seed = rank_seed(cfg, rank)
    gs = make_graph_set(cfg, seed=seed)
    inp = medusa.upload(gs, dev)
    stream = torch.cuda.current_stream(dev)
    slots = medusa.alloc_slots(gs.n_words, dev)
    dst = torch.empty_like(inp["words"])
    fout = torch.empty(gs.n_nodes, dtype=torch.int64, device=dev)
    rep = torch.empty(8, dtype=torch.int64, device=dev)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    scrub = torch.empty(max(2 * l2, 256 << 20) // 4, dtype=torch.int32, device=dev)

    def step():
        medusa.kernel_table_set(inp["table"])  # (independent of the analysis)
        medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], out=slots)
        medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                       dst=dst, func_out=fout, report=rep)

    def barrier():
        torch.cuda.synchronize(dev)
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    for i in range(max(args.warmup, 3)):
        scrub.fill_(i)
        step()
    torch.cuda.synchronize(dev)
    assert int(medusa.report_numpy(rep)[0]) == 0, "restore reported validation failures"
    n_slots = slots.n_slots

    # ---- the step as one CUDA graph: kernel_table_set -> materialize_async ->
    #      restore(slot count from the table): the same kernels, no host round trip
    res = torch.zeros(2, dtype=torch.int64, device=dev)
    gdst = torch.empty_like(inp["words"])
    gfout = torch.empty(gs.n_nodes, dtype=torch.int64, device=dev)
    grep = torch.empty(8, dtype=torch.int64, device=dev)

    def step_async():
        medusa.kernel_table_set(inp["table"])  # (independent of the analysis)
        medusa.materialize_async(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], out=slots, result=res)
        medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                       dst=gdst, func_out=gfout, report=grep, from_table=True)

    graph = torch.cuda.CUDAGraph(keep_graph=True)
    with torch.cuda.graph(graph):
        step_async()
    kernels_per_step = graph_kernel_nodes(graph)  # every kernel node of the step is libmedusa's
    graph.instantiate()
    for _ in range(3):
        graph.replay()
    torch.cuda.synchronize(dev)

    # ---- timed region: K steps, L2 scrubbed (2x L2 write) before each --------------
    sampler = ClockSampler(local)
    for i in range(20):  # bring clocks up before the timed steps
        scrub.fill_(i)

    def timed(fn, sampler=None):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        barrier()
        for k in range(args.steps):
            scrub.fill_(k)
            ev[k][0].record(stream)
            fn()
            ev[k][1].record(stream)
        if sampler is not None:
            sampler.poll_until(ev[-1][1])
        barrier()
        return [a.elapsed_time(b) for a, b in ev]

    step_ms = timed(graph.replay, sampler)  # the headline
    clocks = sampler.stop()
    st_, ns_ = medusa.mat_result(res)
    assert st_ == 0 and ns_ == n_slots, (st_, ns_)
    assert int(medusa.report_numpy(grep)[0]) == 0 and torch.equal(gdst, dst) and torch.equal(gfout, fout)
    head_parity, head_slot_id = oracle_parity(gs, slots, n_slots, gdst, gfout, grep)  # this rank's instance vs the CPU oracle
    assert head_parity["ok"], head_parity
    scratch = medusa.scratch_bytes()
    sync_ms = timed(step)  # the same path through the synchronous API (host round trip after materialize)
    # the same K steps again with every libmedusa launch bracketed by events on its
    # stream: per-kernel durations for the roofline and the breakdown
    def step_queued():
        # as step(), with a device spin (~0.2 ms) queued before the analysis and one
        # (~0.1 ms) between the analysis (whose slot-count read-back leaves the GPU
        # idle) and the restore: the host has enqueued each call's launches and
        # events before the GPU reaches them, so the launch events see device time,
        # not the host's launch latency
        medusa.kernel_table_set(inp["table"])
        torch.cuda._sleep(400000)
        medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], out=slots)
        torch.cuda._sleep(200000)
        medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                       dst=dst, func_out=fout, report=rep)

    medusa.timing_enable(True)
    inst_ms = timed(step_queued)
    launches = medusa.timing_read(1 << 20)
    medusa.timing_enable(False)
    total_ms = sum(step_ms)
    max_ms = max_over_ranks(total_ms, dist, dev)
    nodes_total = gs.n_nodes * args.steps * ws
    value = nodes_total / (max_ms / 1e3)

    # per-kernel device time inside the timed region (events on the launch stream)
    per = {}
    for name, ms in launches:
        d = per.setdefault(name, [0, 0.0])
        d[0] += 1
        d[1] += ms
    counts = path_counts(gs, head_slot_id)
    alg = algorithmic_bytes(gs, n_slots, gs.table.size, counts)
    peak, peak_src = measured_peak()
    traffic = load_traffic(cfg)
    kernels = {}
    for name, (cnt, ms) in sorted(per.items(), key=lambda kv: -kv[1][1]):
        avg = ms / cnt
        entry = {"launches": cnt, "avg_us": 1e3 * avg, "share_of_step": ms / sum(v[1] for v in per.values())}
        if name in alg:
            entry["alg_bytes"] = alg[name]
            entry["GB/s"] = alg[name] / (avg / 1e3) / 1e9
        if traffic.get(name):
            entry["dram_bytes_ncu"] = traffic[name]
        kernels[name] = entry
    dom = max((n for n in per if n in alg), key=lambda n: per[n][1])
    dom_avg_s = per[dom][1] / per[dom][0] / 1e3
    achieved = alg[dom] / dom_avg_s / 1e9
    rl = {"kernel": dom, "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
          "frac": achieved / peak, "traffic": traffic.get(dom), "peak_source": peak_src,
          "alg_bytes_per_launch": alg[dom]}
    inst = traffic.get("_inst", {}).get(dom)
    if inst:  # the instruction-issue view: warp instructions per launch from the
        # committed ncu launch list / this run's launch duration, against 4 schedulers x SMs x clock
        sm_count = torch.cuda.get_device_properties(dev).multi_processor_count
        issue_peak = 4 * sm_count * 1.965e9 / 1e12  # T warp-instructions/s at the 1965 MHz max SM clock
        rl["issue"] = {"warp_inst_per_launch": inst, "achieved": inst / dom_avg_s / 1e12, "peak": issue_peak,
                       "unit": "T warp-inst/s", "frac": inst / dom_avg_s / 1e12 / issue_peak}
    if dom == "mat_classify":
        rl["note"] = ("k_classify reads each word once (TMA) but its time goes to dependent work behind CTA "
                      "barriers (node starts, mortal-tree query, window loads, live masks) and the per-candidate "
                      "lookups: latency- and issue-bound, not HBM-bound; stall breakdown in "
                      "profiles/r2_classify_stalls.txt, DESIGN.md §6")
    # the whole step against the roofline: SURVEY.md §8(d)'s algorithmic bytes of the
    # path (K1+K2 + K3+K4) over the device-timed step
    step_alg = alg["mat_classify"] + alg["restore"]
    step_s = max_ms / args.steps / 1e3
    rl["whole_step"] = {"alg_bytes": step_alg, "ms_per_step": step_s * 1e3, "achieved": step_alg / step_s / 1e9,
                        "frac": step_alg / step_s / 1e9 / peak, "unit": "GB/s"}
    rst = per["restore"]
    restore_avg_s = rst[1] / rst[0] / 1e3
    relocate = {"kernel": "restore", "GB/s": alg["restore"] / restore_avg_s / 1e9,
                "frac_of_peak": alg["restore"] / restore_avg_s / 1e9 / peak,
                "nodes_per_s": gs.n_nodes / restore_avg_s, "avg_us": restore_avg_s * 1e6,
                "traffic": traffic.get("restore")}
    mat_s = sum(v[1] for k, v in per.items() if k.startswith("mat_")) / args.steps / 1e3

    # ---- sustained relocate: ONE restore call over R concatenated
    #      replicas of the workload (>= 1 GB of traffic, so launch, ramp and drain
    #      amortize and nothing stays in L2); materialized once, untimed ----
    sus = None
    if args.sustained > 0:
        from workloads.graphset import replicate
        R = args.sustained
        big = replicate(gs, R)
        binp = medusa.upload(big, dev)
        bslots = medusa.materialize(binp["words"], binp["node_off"], binp["node_t"], binp["allocs"])
        medusa.kernel_table_set(binp["table"])
        bdst = torch.empty_like(binp["words"])
        bfout = torch.empty(big.n_nodes, dtype=torch.int64, device=dev)
        for _ in range(2):
            medusa.restore(binp["words"], bslots, binp["old_base"], binp["new_base"], binp["new_size"],
                           binp["func_id"], dst=bdst, func_out=bfout, report=rep)
        torch.cuda.synchronize(dev)
        assert int(medusa.report_numpy(rep)[0]) == 0
        balg = algorithmic_bytes(big, bslots.n_slots, big.table.size)["restore"]
        reps = 10
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        scrub.fill_(7)
        e0.record(stream)
        for _ in range(reps):
            medusa.restore(binp["words"], bslots, binp["old_base"], binp["new_base"], binp["new_size"],
                           binp["func_id"], dst=bdst, func_out=bfout, report=rep)
        e1.record(stream)
        torch.cuda.synchronize(dev)
        s = e0.elapsed_time(e1) / 1e3 / reps
        sus = {"replicas": R, "nodes": big.n_nodes, "words": big.n_words, "alg_bytes": balg,
               "avg_ms": s * 1e3, "GB/s": balg / s / 1e9, "frac_of_peak": balg / s / 1e9 / peak,
               "nodes_per_s": big.n_nodes / s,
               "note": f"{reps} back-to-back medusa_restore calls, each over {R} concatenated replicas "
                       f"({balg / 1e9:.2f} GB algorithmic traffic per call)"}
        medusa.kernel_table_set(inp["table"])
        del binp, bslots, bdst, bfout, big
        torch.cuda.empty_cache()

    # ---- relocate in place (the online phase patches the loaded image): the image is
    #      restored old -> new, then new -> old, alternately (every call a real,
    #      validated relocation); L2 scrubbed before each call ----
    inpl = bench_inplace(medusa, gs, inp, slots, dev, stream, scrub, args.steps, peak, alg, args.sustained)

    # ---- copy-free buffer contents restoration (§4.3): plan
    #      from this step's table, the permanent buffers given real addresses ----
    buf = bench_buffers(medusa, gs, inp, slots, dev, stream, scrub, args.steps, peak) if args.buffers else None

    # ---- end to end: pinned host buffers -> H2D -> whole path -> D2H of results ----
    # A step's inputs are staged in one pinned host buffer (each array at a 256-B
    # aligned offset) and go up with one copy; its results (restored words, kernel
    # addresses, report, outcome) sit in one device buffer and come down with one
    # copy (nine separate input copies cost ~0.13 ms per step: tools/e2e_probe.py).
    h = medusa.host_arrays(gs)

    def layout(specs):
        lay, off = {}, 0
        for name, dt, shape in specs:
            nb = int(np.prod(shape)) * torch.empty(0, dtype=dt).element_size()
            lay[name] = (off, nb, dt, shape)
            off = (off + nb + 255) & ~255
        return lay, off

    def views(buf, lay):
        return {k: buf[o:o + nb].view(dt).view(shape) for k, (o, nb, dt, shape) in lay.items()}

    in_lay, in_bytes = layout([(k, torch.from_numpy(v).dtype, tuple(v.shape)) for k, v in h.items()])
    out_lay, out_bytes = layout([("dst", torch.int64, (gs.n_words,)), ("fout", torch.int64, (gs.n_nodes,)),
                                 ("rep", torch.int64, (8,)), ("res", torch.int64, (2,))])
    h_in = torch.empty(in_bytes, dtype=torch.uint8).pin_memory()
    for k, v in views(h_in, in_lay).items():
        v.copy_(torch.from_numpy(h[k]))
    h2d, d2h = in_bytes, out_bytes

    def make_set():
        S = dict(d_in_buf=torch.empty(in_bytes, dtype=torch.uint8, device=dev),
                 d_out_buf=torch.zeros(out_bytes, dtype=torch.uint8, device=dev),
                 h_out_buf=torch.empty(out_bytes, dtype=torch.uint8).pin_memory(),
                 slots=medusa.alloc_slots(gs.n_words, dev),
                 ev_in=torch.cuda.Event(), ev_cp=torch.cuda.Event(), ev_out=torch.cuda.Event())
        S["d_in"], S["d_out"], S["h_out"] = views(S["d_in_buf"], in_lay), views(S["d_out_buf"], out_lay), \
            views(S["h_out_buf"], out_lay)
        return S

    ser = make_set()

    def e2e_step():
        d, o = ser["d_in"], ser["d_out"]
        ser["d_in_buf"].copy_(h_in, non_blocking=True)
        medusa.kernel_table_set(d["table"])
        medusa.materialize(d["words"], d["node_off"], d["node_t"], d["allocs"], out=ser["slots"])
        medusa.restore(d["words"], ser["slots"], d["old_base"], d["new_base"], d["new_size"],
                       d["func_id"], dst=o["dst"], func_out=o["fout"], report=o["rep"])
        ser["h_out_buf"].copy_(ser["d_out_buf"], non_blocking=True)

    for _ in range(2):
        e2e_step()
    barrier()
    e2e_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for k in range(args.steps):
        e2e_ev[k][0].record(stream)
        e2e_step()
        e2e_ev[k][1].record(stream)
    barrier()
    e2e_serial_ms = sum(a.elapsed_time(b) for a, b in e2e_ev)
    out_h, fout_h = ser["h_out"]["dst"], ser["h_out"]["fout"]
    assert np.array_equal(out_h.numpy().view(np.uint64), medusa.to_numpy_u64(dst))
    assert int(ser["h_out"]["rep"][0].item()) == 0

    # pipelined end to end (the same public API calls, asynchronous variant): step k's
    # inputs go up on a copy stream, its analysis + restore run on the compute stream,
    # its results come down on a second copy stream, with two buffer sets so that
    # step k+1's upload and step k-1's download overlap step k's kernels.  Every step
    # still copies its full inputs in and its full results out.
    s_in, s_cp, s_out = torch.cuda.Stream(dev), torch.cuda.Stream(dev), torch.cuda.Stream(dev)
    sets = [make_set() for _ in range(args.e2e_sets)]

    def e2e_pipelined(n):
        for k in range(n):
            S = sets[k % len(sets)]
            with torch.cuda.stream(s_in):
                if k >= len(sets):
                    s_in.wait_event(S["ev_cp"])  # the set's inputs are no longer read
                S["d_in_buf"].copy_(h_in, non_blocking=True)
                S["ev_in"].record(s_in)
            with torch.cuda.stream(s_cp):
                s_cp.wait_event(S["ev_in"])
                if k >= len(sets):
                    s_cp.wait_event(S["ev_out"])  # the set's outputs have been read back
                d, o = S["d_in"], S["d_out"]
                medusa.kernel_table_set(d["table"], stream=s_cp)
                medusa.materialize_async(d["words"], d["node_off"], d["node_t"], d["allocs"], out=S["slots"],
                                         result=o["res"], stream=s_cp)
                medusa.restore(d["words"], S["slots"], d["old_base"], d["new_base"], d["new_size"], d["func_id"],
                               dst=o["dst"], func_out=o["fout"], report=o["rep"], stream=s_cp, from_table=True)
                S["ev_cp"].record(s_cp)
            with torch.cuda.stream(s_out):
                s_out.wait_event(S["ev_cp"])
                S["h_out_buf"].copy_(S["d_out_buf"], non_blocking=True)
                S["ev_out"].record(s_out)

    e2e_pipelined(2)
    barrier()
    pa, pb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    pa.record(s_in)
    t_host = time.perf_counter()
    e2e_pipelined(args.steps)
    t_host = time.perf_counter() - t_host
    for S in sets:
        s_out.wait_event(S["ev_out"])
    pb.record(s_out)
    barrier()
    e2e_ms = pa.elapsed_time(pb)
    print(f"e2e pipelined: {args.e2e_sets} buffer sets, host enqueue {1e3 * t_host / args.steps:.3f} ms/step, "
          f"device {e2e_ms / args.steps:.3f} ms/step", file=sys.stderr)
    for S in sets:  # every set's last step: status, slot count, restored words, handles, report
        ho = S["h_out"]
        assert int(ho["res"][0].item()) & 0xFFFFFFFF == 0 and int(ho["res"][1].item()) == n_slots
        assert torch.equal(ho["dst"], out_h) and torch.equal(ho["fout"], fout_h)
        assert int(ho["rep"][0].item()) == 0
    e2e_value = nodes_total / (max_over_ranks(e2e_ms, dist, dev) / 1e3)
    e2e_serial = nodes_total / (max_over_ranks(e2e_serial_ms, dist, dev) / 1e3)

    # ---- C5: one Llama-2-13B-shaped instance per GPU, all GPUs at once ----
    c5 = bench_c5(medusa, args, rank, dev, stream, scrub, barrier, peak) if args.c5 else None
    if c5 is not None:
        assert c5["parity"]["ok"], c5["parity"]
    per_rank = gather_to_all({"rank": rank, "device": torch.cuda.get_device_name(dev), "seed": seed,
                              "sum_ms": total_ms, "headline_parity": head_parity, "c5": c5}, dist)
    multi = {"collective": "none: ranks meet only in a host-side gloo group (barriers, max of device times, "
                           "this gather); no NCCL, nothing crosses GPUs",
             "headline_per_rank": [{"rank": r["rank"], "seed": r["seed"], "ms_per_step": r["sum_ms"] / args.steps,
                                    "parity": r["headline_parity"]} for r in per_rank]}
    if c5 is not None:
        c5s = [r["c5"] for r in per_rank]
        c5_max_ms = max(c["sum_ms"] for c in c5s)
        multi["c5"] = {
            "workload": "C5: one Llama-2-13B-shaped instance per GPU (16,150 nodes, seed 100 + rank), whole path as "
                        "one CUDA graph per step, L2 scrubbed before each step, all GPUs timed at once",
            "aggregate_nodes_per_s": sum(c["nodes"] for c in c5s) * args.steps / (c5_max_ms / 1e3),
            "ms_per_step": c5_max_ms / args.steps,
            "per_gpu": c5s}

    # ---- CPU baseline: the oracle as it stands, rank 0 at N=1 only ----
    cpu = None
    if ws == 1 and not args.no_cpu_baseline:
        ge.build_oracle()
        import oracle
        reps, t_mat, t_res, t0 = 0, 0.0, 0.0, time.perf_counter()
        while time.perf_counter() - t0 < args.cpu_seconds:
            t1 = time.perf_counter()
            m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
            t2 = time.perf_counter()
            oracle.restore(gs.words, m["slot_g"], m["slot_id"], m["slot_off"], gs.allocs["base"], gs.new_base,
                           gs.new_size, gs.func_id, gs.table)
            t_mat += t2 - t1
            t_res += time.perf_counter() - t2
            reps += 1
        t_cpu = t_mat + t_res
        gpu_mat_s = mat_s
        gpu_res_s = restore_avg_s
        cpu = {"value": gs.n_nodes * reps / t_cpu, "unit": "nodes/s", "cores": 1, "kind": "oracle",
               "materialize_nodes_per_s": gs.n_nodes * reps / t_mat,
               "restore_nodes_per_s": gs.n_nodes * reps / t_res,
               "gpu_speedup": {"whole_path": value / (gs.n_nodes * reps / t_cpu),
                               "materialize": (gs.n_nodes / gpu_mat_s) / (gs.n_nodes * reps / t_mat),
                               "restore": (gs.n_nodes / gpu_res_s) / (gs.n_nodes * reps / t_res)},
               "sample": f"the full per-rank {cfg} set, {reps} passes (materialize + restore), "
                         f"single-threaded oracle/oracle.cpp; host has {os.cpu_count()} cores ({cpu_model()})"}
        v, vm, vr, thr, preps = oracle_all_cores(oracle, gs, args.cpu_seconds / 2)
        cpu["all_cores"] = {"value": v, "unit": "nodes/s", "cores": thr, "materialize_nodes_per_s": vm,
                            "restore_nodes_per_s": vr, "gpu_speedup_whole_path": value / v,
                            "sample": f"the same set, {preps} passes; the unchanged oracle on {thr} threads "
                                      "(node ranges for materialize, word ranges for restore; outputs equal "
                                      "the single-threaded run); time of the split / merge in numpy excluded"}

    if rank == 0:
        line = {
            "metric": "graph nodes restored/sec (materialize + restore, whole hot path)",
            "value": value, "unit": "nodes/s", "n_gpus": ws, "steps": args.steps, "warmup": max(args.warmup, 3),
            "ms_per_step": max_ms / args.steps, "higher_is_better": True,
            "step_ms_p10_p50_p90": [float(np.percentile(step_ms, q)) for q in (10, 50, 90)], "scaling": "weak", "vs_baseline": None,
            "dtype": "u64", "data": "synthetic",
            "config": config_dict(cfg, desc, gs, n_slots, rank_seed(cfg, 0), ws),
            "multi_gpu": multi,
            "path_counts": counts,
            "scratch": {"bytes": scratch, "bytes_per_word": scratch / gs.n_words,
                        "note": "library-owned materialize scratch of this device after the headline workload "
                                "(medusa_scratch_bytes)"},
            "roofline": rl,
            "relocate": relocate,
            "materialize_ms": mat_s * 1e3,
            "kernels": kernels,
            "sustained_relocate": sus,
            "relocate_in_place": inpl,
            "buffers": buf,
            "cpu_baseline": cpu,
            "paper_context": PAPER_CONTEXT,
            "e2e": {"value": e2e_value, "unit": "nodes/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                    "mode": "pipelined: inputs up (copy stream) / materialize_async + restore (compute stream) / "
                            "results down (copy stream), two buffer sets; every step copies all its inputs (one "
                            "pinned staging buffer, one H2D copy) and all its results (one device buffer, one D2H "
                            "copy); timed from the first upload to the last download",
                    "serial_value": e2e_serial,
                    "serial_mode": "one step at a time: H2D, medusa_materialize (host round trip), "
                                   "medusa_restore, D2H, on one stream"},
            "gpu_launches": kernels_per_step * args.steps,
            "graph_step": "one CUDA graph per step: medusa_kernel_table_set, medusa_materialize_async, "
                          f"medusa_restore(MEDUSA_N_SLOTS_FROM_TABLE); {kernels_per_step} libmedusa kernels per step "
                          "(kernel nodes of the captured graph; the instrumented synchronous pass launched "
                          f"{len(launches) // max(args.steps, 1)} per step: no k_result)",
            "sync_api_ms_per_step": max_over_ranks(sum(sync_ms), dist, dev) / args.steps,
            "instrumented_ms_per_step": sum(inst_ms) / args.steps,
            "instrumented_note": "per-kernel events, branches serialized, device spins queued before the analysis "
                                 "(~0.2 ms) and before the restore (~0.1 ms) so no event waits for the host; "
                                 "instrumented_ms_per_step includes the spins (share_of_step = share of the summed "
                                 "kernel times, as in the ncu launch list)",
            "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=None, help="GPUs (default: WORLD_SIZE under torchrun, else 1)")
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", choices=sorted(WORKLOADS), default="all10")
    ap.add_argument("--sustained", type=int, default=32, help="replicas in the sustained-relocate call (0: skip)")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-sets", type=int, default=2, help="buffer sets in the pipelined end-to-end leg")
    ap.add_argument("--no-buffers", dest="buffers", action="store_false")
    ap.add_argument("--c5-sustained", type=int, default=256,
                    help="replicas of the per-GPU C5 instance in its sustained-relocate call (0: skip)")
    ap.add_argument("--no-c5", dest="c5", action="store_false", help="skip the per-GPU C5 block")
    ap.add_argument("--selftest-plumbing", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args()
    ws_env = os.environ.get("WORLD_SIZE")
    if args.gpus is None:
        args.gpus = int(ws_env) if ws_env else 1
    if ws_env is not None and int(ws_env) != args.gpus:
        raise SystemExit(f"bench.py --gpus {args.gpus} under a launcher with WORLD_SIZE={ws_env}")
    if args.impl == "reference":
        run_reference(args)  # rank 0 only: the CPU oracle (other ranks exit at once)
    elif ws_env is None and args.gpus > 1:
        spawn_ranks(args, n_visible=args.gpus if args.selftest_plumbing else None)
    elif args.selftest_plumbing:
        plumbing_selftest(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
