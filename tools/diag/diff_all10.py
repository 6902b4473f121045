"""Diagnostic: materialize ALL10 (optionally after other calls) and report which
slots differ from the oracle (chunk, word, id, I or mortal)."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import oracle
import paper_conf_asplos_zengxgcl25_b200 as medusa
from workloads import make_graph_set, ALLOC_DTYPE, T_NEVER
from tests.tiny import tiny_trace

DEV = torch.device("cuda:0")
gs = make_graph_set("all10")
m = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)
mask, cb, rec = oracle.pack(m, gs.n_words)
inp = medusa.upload(gs, DEV)
tl = int(gs.node_t[-1])
isI = (gs.allocs["size"] > 0) & (gs.allocs["t_alloc"] < tl) & (tl < gs.allocs["t_free"])


def run(tag):
    s = medusa.materialize(inp["words"], inp["node_off"], inp["node_t"], inp["allocs"])
    gm = s.mask.cpu().numpy().view(np.uint32)
    bits_g = np.unpackbits(gm.view(np.uint8), bitorder="little")[: gs.n_words].astype(bool)
    bits_o = m["is_slot"].astype(bool)
    miss = np.flatnonzero(bits_o & ~bits_g)
    extra = np.flatnonzero(bits_g & ~bits_o)
    ids = m["id"][miss]
    print(tag, "n_slots", s.n_slots, m["n_slots"], "missing", miss.size, "extra", extra.size,
          "missing I", int(isI[ids].sum()), "chunks", np.unique(miss // 2048)[:20], "ids", ids[:10], flush=True)


t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(DEV)
for k in range(3):
    run(f"fresh{k}")
for mode in sys.argv[1:]:
    if mode == "tiny":
        for seed in range(50):
            words, off, nt, allocs = tiny_trace(seed * 7)
            aa = np.ascontiguousarray(allocs).view(np.int64).reshape(-1, 3) if allocs.size else np.zeros((0, 3), np.int64)
            try:
                medusa.materialize(t(words, np.int64), t(off, np.int64), t(nt, np.int32), torch.from_numpy(aa).to(DEV))
            except medusa.MedusaError:
                pass
    if mode == "bad":
        b = 0x7F00_0000_0000
        w = np.uint64(b) + np.arange(4096, dtype=np.uint64) * np.uint64(8)
        A = np.array([(b, 8 * 4096, 1, T_NEVER)], dtype=ALLOC_DTYPE)
        aa = torch.from_numpy(np.ascontiguousarray(A).view(np.int64).reshape(-1, 3)).to(DEV)
        for off in ([0, 3000, 100, 4096], [0, 3000, 5000, 4096]):
            try:
                medusa.materialize(t(w, np.int64), t(np.array(off, np.uint64), np.int64), t(np.array([2, 3, 4], np.uint32), np.int32), aa)
            except medusa.MedusaError as e:
                print("bad", e.status)
    run(f"after_{mode}")
    run(f"after_{mode}_2")
