"""Real-capture check with a summary line: a PyTorch
decoder captured into a CUDA graph -> parameter image + allocation trace ->
medusa_materialize -> replayed allocations -> medusa_restore -> clone of the
graph with the restored parameters -> bit-identical output.
usage: python tools/real_capture_demo.py"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_asplos_zengxgcl25_b200 as medusa  # noqa: E402
from workloads.capture import real_graph  # noqa: E402

r = real_graph.end_to_end(torch, medusa)
print(json.dumps({
    "graphs": r["n_graphs"], "graph_nodes": r["n_nodes"], "kernel_nodes": r["n_kernel"], "other_nodes": r["n_other"],
    "distinct_kernels": len(r["kernel_names"]), "words": int(r["words"].size), "allocations": int(len(r["allocs"])),
    "allocated_before_capture": r["n_pre"], "slots": r["slots"].n_slots,
    "slot_words_share": r["slots"].n_slots / max(int(r["words"].size), 1),
    "restore_report_bad": int(r["report"][0]), "outputs_bit_identical": all(bool(torch.equal(a, b)) for a, b in zip(r["outs_b"], r["refs"])),
    "buffer_classes": {k: int((r["buf_class"] == v).sum()) for k, v in (("unused", 0), ("param", 1), ("temp", 2), ("perm", 3))},
    "permanent_buffers": r["n_perm"], "saved_blob_bytes": r["blob_bytes"],
    "outputs_equal_without_permanent_contents": [bool(torch.equal(a, b)) for a, b in zip(r["outs_unrestored"], r["refs"])],
    "kernels_sample": sorted(r["kernel_names"])[:8],
}, indent=1))
