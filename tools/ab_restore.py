"""A/B of restore-kernel variants on B200: builds libmedusa with each
-DMEDUSA_RESTORE_CPB value (chunks per CTA), times one medusa_restore over the
ALL10 set (L2 scrubbed before each call) and over 32 replicas (sustained), and
checks every variant's output against the first one.

  python tools/ab_restore.py [--cpb 1 2 4] [--reps 30]
"""
import argparse
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import __graft_entry__ as g  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cpb", type=int, nargs="+", default=[1, 2, 4])
    ap.add_argument("--reps", type=int, default=30)
    ap.add_argument("--replicas", type=int, default=32)
    ap.add_argument("--inplace", action="store_true", help="variants of the in-place kernel (MEDUSA_RESTORE_CPB_IP)")
    ap.add_argument("--defines", nargs="+", help="variants given as preprocessor defines (e.g. MEDUSA_RESTORE_EARLY=0)")
    args = ap.parse_args()
    if args.defines:
        names = args.defines
        libs = {d: g.build_medusa(out=os.path.join(ROOT, "tools", f"libmedusa_{d.replace('=', '_')}.so"), defines=(d,))
                for d in names}
    else:
        names = args.cpb
        libs = {c: g.build_medusa(out=os.path.join(ROOT, "tools", f"libmedusa_cpb{c}.so"),
                                  defines=(f"MEDUSA_RESTORE_CPB{'_IP' if args.inplace else ''}={c}",))
                for c in args.cpb}
    import paper_conf_asplos_zengxgcl25_b200 as medusa
    from bench import algorithmic_bytes
    from workloads import make_graph_set
    from workloads.graphset import replicate
    dev = torch.device("cuda:0")
    gs = make_graph_set("all10")
    big = replicate(gs, args.replicas)
    sets = []
    for x in (gs, big):
        inp = medusa.upload(x, dev)
        sl = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
        sets.append((x, inp, sl, algorithmic_bytes(x, sl.n_slots, x.table.size)["restore"]))
    scrub = torch.empty(256 << 20 >> 2, dtype=torch.int32, device=dev)
    ref = None
    for c in names:
        path = libs[c]
        medusa._lib = None
        medusa.LIB_PATH = path
        medusa.lib()
        line = [c if args.defines else f"CPB{'_IP' if args.inplace else ''}={c}"]
        for si, (x, inp, sl, alg) in enumerate(sets):
            medusa.kernel_table_set(inp["table"])
            dst = inp["words"].clone() if args.inplace else torch.empty_like(inp["words"])
            fout = torch.empty(x.n_nodes, dtype=torch.int64, device=dev)
            rep = torch.empty(8, dtype=torch.int64, device=dev)
            src = dst if args.inplace else inp["words"]
            # in place: identity relocation (old == new) so that every replay is a valid restore
            nb = inp["old_base"] if args.inplace else inp["new_base"]
            run = lambda: medusa.restore(src, sl, inp["old_base"], nb, inp["new_size"],
                                         inp["func_id"], dst=dst, func_out=fout, report=rep)
            for _ in range(3):
                run()
            graph = torch.cuda.CUDAGraph()  # device time only: no host launch overhead inside the events
            with torch.cuda.graph(graph):
                run()
            ts = []
            for k in range(args.reps if si == 0 else 5):
                scrub.fill_(k)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                graph.replay()
                b.record()
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            t = statistics.median(ts) / 1e3
            assert int(medusa.report_numpy(rep)[0]) == 0
            if si == 0 and not args.inplace:
                h = (dst.cpu().numpy().copy(), fout.cpu().numpy().copy())
                if ref is None:
                    ref = h
                assert np.array_equal(h[0], ref[0]) and np.array_equal(h[1], ref[1]), f"{c}: output differs"
            line.append(f"{'all10' if si == 0 else 'x%d' % args.replicas}: {t * 1e6:8.1f} us "
                        f"{alg / t / 1e9:6.0f} GB/s")
        print("  ".join(line), flush=True)


if __name__ == "__main__":
    main()
