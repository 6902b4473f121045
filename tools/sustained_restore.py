"""One restore call over R concatenated replicas of a workload (SURVEY.md §8(d)
sustained mode), out of place and in place, for an ncu capture of the sustained
relocate pass: `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,
gpu__time_duration.sum -k regex:restore python tools/sustained_restore.py`.
Prints the algorithmic bytes of each call and checks the report (diagnostic)."""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="all10")
    ap.add_argument("--replicas", type=int, default=32)
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    import __graft_entry__ as g
    g.build_medusa()
    import bench
    import paper_conf_asplos_zengxgcl25_b200 as medusa
    from workloads import make_graph_set
    from workloads.graphset import replicate
    dev = torch.device("cuda:0")
    big = replicate(make_graph_set(args.workload), args.replicas)
    inp = medusa.upload(big, dev)
    sl = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    medusa.kernel_table_set(inp["table"])
    dst = torch.empty_like(inp["words"])
    rep = torch.empty(8, dtype=torch.int64, device=dev)
    alg = bench.algorithmic_bytes(big, sl.n_slots, big.table.size)
    out = {"workload": f"{args.workload} x{args.replicas}", "words": big.n_words, "nodes": big.n_nodes,
           "slots": sl.n_slots, "alg_bytes_out_of_place": alg["restore"], "alg_bytes_in_place": alg["restore_inplace"]}
    for _ in range(args.reps):  # out of place
        medusa.restore(inp["words"], sl, inp["old_base"], inp["new_base"], inp["new_size"], inp["func_id"], dst=dst,
                       report=rep)
    torch.cuda.synchronize()
    out["report_out_of_place"] = int(medusa.report_numpy(rep)[0])
    buf = inp["words"].clone()
    fwd = (inp["old_base"], inp["new_base"])
    for k in range(args.reps):  # in place, old -> new -> old ...
        ob, nb = fwd if k % 2 == 0 else fwd[::-1]
        medusa.restore(buf, sl, ob, nb, inp["new_size"], inp["func_id"], dst=buf, report=rep)
    torch.cuda.synchronize()
    out["report_in_place"] = int(medusa.report_numpy(rep)[0])
    print(json.dumps(out))


if __name__ == "__main__":
    main()
