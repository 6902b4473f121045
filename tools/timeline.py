"""Per-CTA timeline of one graph-captured step (diagnostic; not part of the product).

Builds tools/libmedusa_tl.so with -DMEDUSA_TIMELINE (thread 0 of every CTA
stamps %globaltimer at start and end), replays the bench step (materialize_async
-> kernel_table_set -> restore) K times with an L2 scrub before each, and prints
per kernel/role: CTA count, first start / last end relative to the step start,
CTA duration percentiles, and the idle gap before each kernel.

usage: python tools/timeline.py [--workload all10] [--steps 5]
"""
import argparse
import ctypes
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import __graft_entry__ as g  # noqa: E402

NAMES = {(1, 0): "trace/nodes", (1, 1): "trace/allocs", (1, 2): "trace/last-scan",
         (2, 0): "isort", (2, 1): "prepare/scatter", (3, 0): "rank",
         (4, 0): "classify",
         (5, 0): "emit", (8, 0): "check_mm", (9, 0): "check", (10, 0): "iresolve", (6, 0): "report_init", (7, 0): "restore/words", (7, 1): "restore/gather",
         (1, 20): " allocs:load+checks", (1, 21): " allocs:stage", (1, 22): " allocs:tree+I",
         (1, 23): " last:fence", (1, 24): " last:scan-c", (1, 25): " last:scan-b",
         (3, 40): " rank:pdl-wait", (3, 41): " rank:staging", (3, 42): " rank:search+red", (3, 43): " rank:ticket",
         (3, 44): " rank:i-entries", (2, 30): " isort:bitonic", (2, 31): " isort:merges",
         (4, 10): " cls:A setup", (4, 11): " cls:B starts+cand", (4, 12): " cls:D query", (4, 13): " cls:D live+search",
         (4, 14): " cls:E queue", (4, 15): " cls:E records+queue", (4, 16): " cls:win-load", (4, 17): " cls:sort",
         (7, 2): "restore/in-place", (7, 10): " res:mask+range", (7, 11): " res:records+gathers",
         (7, 12): " res:apply (+word wait)", (7, 13): " res:bulk store",
         (10, 50): " ires:fences+prefix", (10, 51): " ires:queue entry", (10, 52): " ires:fence search+group",
         (10, 53): " ires:entry+mask", (5, 60): " emit:wait", (5, 61): " emit:masks+prefix",
         (5, 62): " emit:popc prefixes", (5, 63): " emit:records"}
REC = np.dtype([("t0", "<u8"), ("t1", "<u8"), ("kernel", "<u4"), ("cta", "<u4"), ("sm", "<u4"), ("tag", "<u4")])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="all10")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--serial", action="store_true",
                    help="every kernel alone (libmedusa's per-launch timing mode: branches serialized)")
    args = ap.parse_args()
    extra = tuple(d for d in os.environ.get("MEDUSA_DEFINES", "").split() if d)  # A/B variants
    tl_path = g.build_medusa(out=os.path.join(ROOT, "tools", "libmedusa_tl" + "".join("_" + d for d in extra) + ".so"),
                             defines=("MEDUSA_TIMELINE",) + extra)
    import paper_conf_asplos_zengxgcl25_b200 as medusa
    from workloads import CONFIGS, make_graph_set
    medusa._lib = None
    medusa.LIB_PATH = tl_path
    L = medusa.lib()
    for sfx in ("mat", "res"):
        getattr(L, f"medusa_tl_attach_{sfx}").argtypes = [ctypes.c_void_p, ctypes.c_uint]
        getattr(L, f"medusa_tl_count_{sfx}").restype = ctypes.c_uint
    dev = torch.device("cuda:0")
    gs = make_graph_set(args.workload, seed=1)
    inp = medusa.upload(gs, dev)
    slots = medusa.alloc_slots(gs.n_words, dev)
    res = torch.zeros(2, dtype=torch.int64, device=dev)
    dst = torch.empty_like(inp["words"])
    fout = torch.empty(gs.n_nodes, dtype=torch.int64, device=dev)
    rep = torch.empty(8, dtype=torch.int64, device=dev)
    medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], out=slots)  # sizes scratch

    def step():
        medusa.kernel_table_set(inp["table"])  # (independent of the analysis)
        medusa.materialize_async(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"], out=slots, result=res)
        medusa.restore(inp["words"], slots, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"],
                       dst=dst, func_out=fout, report=rep, from_table=True)

    cap = 1 << 16
    buf = [torch.zeros(cap * REC.itemsize, dtype=torch.uint8, device=dev) for _ in range(2)]
    step()  # eager once: the kernel table and scratch are allocated outside capture
    torch.cuda.synchronize()
    if args.serial:  # eager steps (per-launch events cannot be captured)
        medusa.timing_enable(True)
        run = step
    else:
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            step()
        run = graph.replay
    scrub = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    for _ in range(3):
        run()
    agg = {}
    spans = []
    ev = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
    for k in range(args.steps):
        L.medusa_tl_attach_mat(ctypes.c_void_p(buf[0].data_ptr()), cap)
        L.medusa_tl_attach_res(ctypes.c_void_p(buf[1].data_ptr()), cap)
        scrub.fill_(k)
        ev[0].record()
        run()
        ev[1].record()
        torch.cuda.synchronize()
        n0, n1 = L.medusa_tl_count_mat(), L.medusa_tl_count_res()
        recs = np.concatenate([buf[0][: n0 * REC.itemsize].cpu().numpy().view(REC),
                               buf[1][: n1 * REC.itemsize].cpu().numpy().view(REC)])
        t_begin = recs["t0"].min()
        spans.append(((recs["t1"].max() - t_begin) / 1e3, ev[0].elapsed_time(ev[1]) * 1e3))
        for key in sorted(set(zip(recs["kernel"].tolist(), recs["tag"].tolist()))):
            r = recs[(recs["kernel"] == key[0]) & (recs["tag"] == key[1])]
            d = (r["t1"] - r["t0"]) / 1e3
            agg.setdefault(key, []).append(((r["t0"].min() - t_begin) / 1e3, (r["t1"].max() - t_begin) / 1e3, len(r),
                                            np.percentile(d, 50), np.percentile(d, 90), d.max()))
    if args.serial:
        medusa.timing_read(1 << 16)
        medusa.timing_enable(False)
    assert medusa.mat_result(res)[0] == 0
    print(f"{args.workload}: step span (first CTA start -> last CTA end) {np.mean([s[0] for s in spans]):.1f} us; "
          f"event time {np.mean([s[1] for s in spans]):.1f} us (incl. launch of the first kernel)")
    print(f"{'kernel/role':18s} {'ctas':>6s} {'start':>8s} {'end':>8s} {'span':>7s} {'p50':>7s} {'p90':>7s} {'max':>7s}  (us)")
    for key, rows in sorted(agg.items(), key=lambda kv: np.mean([r[0] for r in kv[1]])):
        a = np.mean(np.array(rows), axis=0)
        print(f"{NAMES.get(key, str(key)):18s} {a[2]:6.0f} {a[0]:8.1f} {a[1]:8.1f} {a[1]-a[0]:7.1f} {a[3]:7.2f} {a[4]:7.2f} {a[5]:7.2f}")


if __name__ == "__main__":
    main()
