"""Real-capture workload and end-to-end check.

A small decoder (random weights, no network) is captured into a CUDA graph by
PyTorch.  The graph's memory comes from a torch.cuda.MemPool whose segments are
served by the tracing allocator in trace_alloc.cpp, which logs every segment
allocation / free together with the number of nodes the capturing graph held
at that moment: one total order of allocations and kernel launches.
The parameter image is read from the captured graph itself:
cuGraphKernelNodeGetParams gives each kernel node's function and argument
pointers, cuFuncGetParamInfo / cuKernelGetParamInfo the device-side layout
(offset, size) of every argument (Fig. 4d); memset nodes contribute
their destination pointer as a one-word blob.

The "online process" is emulated in the same process (same kernel handles, so
the kernel table of §5 is not exercised here): the allocation sequence is
replayed in a second arena (different addresses), the contents of every
traced segment are copied over (= loading the same weights and inputs), the
first arena is poisoned, and a clone of the graph gets every kernel / memset
node's parameters replaced by the restored image (cuGraphKernelNodeSetParams,
NEXT-2).  Its output must equal, bit for bit, the output the original graph
produced; a pointer the analysis missed would read poisoned memory.

Device-only module (needs a GPU, the CUDA driver bindings and torch).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "libtrace_alloc.so")
SRC = os.path.join(HERE, "trace_alloc.cpp")
T_END = 0xFFFFFFFF


def build(force=False):
    """Compile the tracing allocator (plain C++ against the CUDA runtime)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.run(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-I/usr/local/cuda/include", "-o", LIB, SRC,
                        "-L/usr/local/cuda/lib64", "-lcudart"], check=True, capture_output=True)
    return LIB


def _lib():
    L = ctypes.CDLL(build())
    L.ta_init.argtypes = [ctypes.c_uint64]
    L.ta_init.restype = ctypes.c_int
    L.ta_select.argtypes = [ctypes.c_int]
    L.ta_log.argtypes = [ctypes.c_int]
    L.ta_capture_begin.argtypes = [ctypes.c_int64]
    L.ta_raw_malloc.argtypes = [ctypes.c_uint64]
    L.ta_raw_malloc.restype = ctypes.c_uint64
    L.ta_events.argtypes = [ctypes.POINTER(ctypes.c_int64), ctypes.c_int64]
    L.ta_events.restype = ctypes.c_int64
    L.ta_arena_base.argtypes = [ctypes.c_int]
    L.ta_arena_base.restype = ctypes.c_uint64
    return L


def tiny_decoder(torch, d=256, layers=2, vocab=512, heads=4):
    """A decoder-only transformer with random weights: embedding, per layer RMSNorm
    + causal attention + SwiGLU MLP (cuBLAS GEMMs, softmax, elementwise), lm head."""
    nn = torch.nn

    class Layer(nn.Module):
        def __init__(self):
            super().__init__()
            self.n1 = nn.Parameter(torch.rand(d) + 0.5)
            self.qkv = nn.Linear(d, 3 * d, bias=False)
            self.o = nn.Linear(d, d, bias=False)
            self.n2 = nn.Parameter(torch.rand(d) + 0.5)
            self.up = nn.Linear(d, 4 * d, bias=False)
            self.gate = nn.Linear(d, 4 * d, bias=False)
            self.down = nn.Linear(4 * d, d, bias=False)

        def forward(self, x, mask):
            b, s, _ = x.shape
            h = x * torch.rsqrt(x.pow(2).mean(-1, keepdim=True) + 1e-6) * self.n1
            q, k, v = self.qkv(h).view(b, s, 3, heads, d // heads).permute(2, 0, 3, 1, 4)
            a = torch.softmax((q @ k.transpose(-1, -2)) * (d // heads) ** -0.5 + mask, dim=-1) @ v
            x = x + self.o(a.transpose(1, 2).reshape(b, s, d))
            h = x * torch.rsqrt(x.pow(2).mean(-1, keepdim=True) + 1e-6) * self.n2
            return x + self.down(torch.nn.functional.silu(self.gate(h)) * self.up(h))

    class Model(nn.Module):
        def __init__(self):
            super().__init__()
            self.emb = nn.Embedding(vocab, d)
            self.layers = nn.ModuleList([Layer() for _ in range(layers)])
            self.head = nn.Linear(d, vocab, bias=False)

        def forward(self, ids, mask):
            x = self.emb(ids)
            for layer in self.layers:
                x = layer(x, mask)
            return self.head(x)

    return Model()


def _check(res):
    """The value(s) of a cuda-python call after checking its error code."""
    if not isinstance(res, tuple):
        res = (res,)
    if int(res[0]) != 0:
        raise RuntimeError(f"CUDA call failed: {res[0]}")
    if len(res) == 1:
        return None
    return res[1] if len(res) == 2 else res[1:]


def _param_layout(cu, params):
    """[(offset, size)] of every argument of a kernel node (device-side layout)."""
    out = []
    kern = int(params.kern) if params.kern is not None else 0
    for i in range(4096):
        r = cu.cuKernelGetParamInfo(params.kern, i) if kern else cu.cuFuncGetParamInfo(params.func, i)
        if int(r[0]) != 0:
            break
        out.append((int(r[1]), int(r[2])))
    return out


def capture(torch, batches=(8, 4, 2, 1), seq=16, seed=0, arena_bytes=1 << 30):
    """Process A: build the model in the traced pool and capture one forward per
    batch size into its own CUDA graph, largest first, all graphs sharing one
    memory pool (vLLM's order); replay each once.  Returns the graphs, each
    graph's nodes in launch order, the trace and the reference outputs."""
    from cuda.bindings import driver as cu

    L = _lib()
    if L.ta_init(arena_bytes) != 0:
        raise RuntimeError("tracing allocator: cudaMalloc of the arenas failed")
    alloc = torch.cuda.memory.CUDAPluggableAllocator(build(), "ta_malloc", "ta_free")
    L.ta_select(0)
    L.ta_clear()
    L.ta_log(1)
    pool = torch.cuda.MemPool(alloc.allocator())       # model loading + warm-up
    gpool = torch.cuda.MemPool(alloc.allocator())      # the graphs' private pool (vLLM's graph pool)
    torch.manual_seed(seed)
    with torch.cuda.use_mem_pool(pool):
        model = tiny_decoder(torch).cuda().eval()
        ids = torch.randint(0, 512, (max(batches), seq), device="cuda")  # static input, sliced per graph
        mask = torch.full((seq, seq), float("-inf"), device="cuda").triu(1)
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s), torch.no_grad():
            for b in batches:
                model(ids[:b], mask)
        torch.cuda.current_stream().wait_stream(s)
        torch.cuda.synchronize()
    graphs, outs, magic = [], [], []
    for k, b in enumerate(batches):
        g = torch.cuda.CUDAGraph(keep_graph=True)  # (raw_cuda_graph needs the graph kept)
        L.ta_capture_begin(k)
        with torch.no_grad(), torch.cuda.graph(g, pool=gpool.id):
            if k == 0:
                # one permanent buffer per graph: allocated during the
                # (first) capture before any temporary, never freed, its 4-byte
                # content (a "magic number") written outside the graphs and read by
                # every replay.  (Allocated later, a graph's buffer could reuse a
                # block an earlier graph's temporaries occupy in the shared pool.)
                magic = [torch.empty((), device="cuda") for _ in batches]
            outs.append(model(ids[:b], mask) * magic[k])
        L.ta_capture_end()
        graphs.append(g)
    L.ta_log(0)
    for m in magic:
        m.fill_(1.0)
    for g in graphs:
        g.instantiate()
        g.replay()
    torch.cuda.synchronize()
    refs = [o.detach().cpu().clone() for o in outs]

    # the trace
    n_ev = L.ta_events(None, 0)
    buf = (ctypes.c_int64 * (5 * n_ev))()
    L.ta_events(buf, n_ev)
    ev = np.frombuffer(buf, dtype=np.int64).reshape(n_ev, 5).copy()

    # every graph's nodes in launch order (a stream capture is one chain)
    raw, orders = [], []
    for g in graphs:
        graph = cu.CUgraph(g.raw_cuda_graph())
        n_all = int(cu.cuGraphGetNodes(graph, 0)[2])
        orders.append(_topo(cu, list(cu.cuGraphGetNodes(graph, n_all)[1])))
        raw.append(graph)
    return dict(L=L, pool=pool, gpool=gpool, alloc=alloc, model=model, ids=ids, mask=mask, graph_objs=graphs,
                graphs=raw, nodes=orders, events=ev, outs=outs, refs=refs, magic=magic)


def _topo(cu, nodes):
    """Nodes in dependency order (ties by creation order)."""
    idx = {int(n): k for k, n in enumerate(nodes)}
    indeg = {}
    succ = {int(n): [] for n in nodes}
    for n in nodes:
        r = cu.cuGraphNodeGetDependencies(n, 0)
        cnt = int(r[2])
        deps = list(cu.cuGraphNodeGetDependencies(n, cnt)[1]) if cnt else []
        indeg[int(n)] = len(deps)
        for d_ in deps:
            succ[int(d_)].append(n)
    ready = sorted([n for n in nodes if indeg[int(n)] == 0], key=lambda n: idx[int(n)])
    out = []
    while ready:
        n = ready.pop(0)
        out.append(n)
        for m in succ[int(n)]:
            indeg[int(m)] -= 1
            if indeg[int(m)] == 0:
                ready.append(m)
        ready.sort(key=lambda n: idx[int(n)])
    return out


def parameter_image(cu, graph_nodes):
    """Per kernel / memset node of every graph (graph order, then launch order):
    its blob (8-byte words) and how to rebuild it."""
    recs = []
    for gi, nodes in enumerate(graph_nodes):
        recs += _graph_image(cu, gi, nodes)
    return recs


def _graph_image(cu, gi, nodes):
    recs = []
    for pos, n in enumerate(nodes):
        t = cu.cuGraphNodeGetType(n)[1]
        if t == cu.CUgraphNodeType.CU_GRAPH_NODE_TYPE_KERNEL:
            p = cu.cuGraphKernelNodeGetParams(n)[1]
            layout = _param_layout(cu, p)
            size = max((o + s for o, s in layout), default=0)
            blob = bytearray((size + 7) // 8 * 8)
            kp = ctypes.cast(int(p.kernelParams), ctypes.POINTER(ctypes.c_void_p)) if int(p.kernelParams) else None
            for i, (o, s_) in enumerate(layout):
                if kp is None or not kp[i]:
                    raise RuntimeError("kernel node without kernelParams")
                blob[o:o + s_] = ctypes.string_at(kp[i], s_)
            recs.append(dict(kind="kernel", graph=gi, node=n, pos=pos, params=p, layout=layout, blob=bytes(blob)))
        elif t == cu.CUgraphNodeType.CU_GRAPH_NODE_TYPE_MEMSET:
            p = cu.cuGraphMemsetNodeGetParams(n)[1]
            recs.append(dict(kind="memset", graph=gi, node=n, pos=pos, params=p, blob=int(p.dst).to_bytes(8, "little")))
        else:
            recs.append(dict(kind="other", graph=gi, node=n, pos=pos, type=t))
    return recs


def trace_arrays(ev, recs):
    """medusa inputs from the trace and the node list: allocation records with
    event positions, each kernel / memset node's launch position, and the
    (begin, end) positions of every capture (for medusa_buffers_plan)."""
    from workloads import ALLOC_DTYPE

    n_in = {}
    for r in recs:
        n_in[r["graph"]] = n_in.get(r["graph"], 0) + 1
    node_pos = {}
    t = 1
    cap, emitted = -1, 0

    def emit_until(c, upto):
        nonlocal t, emitted
        while emitted < min(upto, n_in.get(c, 0)):
            node_pos[(c, emitted)] = t
            t += 1
            emitted += 1

    ev_t = []
    caps = []
    for k in range(ev.shape[0]):
        kind = int(ev[k, 0])
        if kind == 3:  # capture `ev[k, 4]` begins
            cap, emitted = int(ev[k, 4]), 0
            caps.append([t, 0])
        elif kind == 4:  # ... ends: all its nodes were launched before what follows
            emit_until(cap, 1 << 62)
            cap = -1
            caps[-1][1] = t
        elif cap >= 0 and int(ev[k, 3]) >= 0:
            emit_until(cap, int(ev[k, 3]))  # nodes captured before this call
        ev_t.append(t)
        t += 1
    allocs = []
    live = {}
    for k in range(ev.shape[0]):
        kind, ptr, size = int(ev[k, 0]), int(ev[k, 1]) & ((1 << 64) - 1), int(ev[k, 2])
        if kind >= 3:
            continue
        if kind == 1:
            live[ptr] = len(allocs)
            allocs.append([ptr, size, ev_t[k], T_END])
        elif ptr in live:
            allocs[live.pop(ptr)][3] = ev_t[k]
    arr = np.zeros(len(allocs), ALLOC_DTYPE)
    for i, (b, s, ta, tf) in enumerate(allocs):
        arr[i] = (b, s, ta, tf)
    used = [r for r in recs if r["kind"] in ("kernel", "memset")]
    words = np.frombuffer(b"".join(r["blob"] for r in used), dtype=np.uint64).copy()
    off = np.zeros(len(used) + 1, np.uint64)
    off[1:] = np.cumsum([len(r["blob"]) // 8 for r in used])
    node_t = np.array([node_pos[(r["graph"], r["pos"])] for r in used], np.uint32)
    capture_t = np.array(caps, np.uint32).reshape(-1, 2)
    return words, off, node_t, arr, used, capture_t


def _alloc_of(allocs, ptr):
    """Ordinal of the latest allocation whose range holds ptr."""
    return int(np.nonzero((allocs["base"] <= ptr) & (ptr < allocs["base"] + allocs["size"]))[0][-1])


def _in_capture(allocs, capture_t, i):
    ta = int(allocs["t_alloc"][i])
    return any(int(b) < ta < int(e) for b, e in capture_t)


def online_bases(L, allocs, events):
    """Replay the (de)allocation sequence in the second arena: new base of every
    allocation ordinal."""
    L.ta_free.argtypes = [ctypes.c_void_p, ctypes.c_ssize_t, ctypes.c_int, ctypes.c_void_p]
    L.ta_select(1)
    new_base = np.zeros(len(allocs), np.uint64)
    moved = {}
    i = 0
    for k in range(events.shape[0]):
        ptr = int(events[k, 1]) & ((1 << 64) - 1)
        if int(events[k, 0]) == 1:
            new_base[i] = L.ta_raw_malloc(int(events[k, 2]))
            moved[ptr] = int(new_base[i])
            i += 1
        elif ptr in moved:
            L.ta_free(ctypes.c_void_p(moved.pop(ptr)), 0, 0, None)
    L.ta_select(0)
    return new_base


def end_to_end(torch, medusa, seed=0):
    """Capture (process A), materialize the real image on the GPU, replay the
    allocations in the second arena, copy the live segments over and poison the
    first arena, restore the image on the GPU, write the restored parameters
    into a clone of the graph and run it.  Returns the facts the test checks."""
    from cuda.bindings import driver as cu
    from cuda.bindings import runtime as rt

    A = capture(torch, seed=seed)
    recs = parameter_image(cu, A["nodes"])
    words, off, node_t, allocs, used, capture_t = trace_arrays(A["events"], recs)
    dev = torch.device("cuda")
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(dev)
    aa = np.ascontiguousarray(allocs).view(np.int64).reshape(-1, 3)
    inp = dict(words=t(words, np.int64), node_off=t(off, np.int64), node_t=t(node_t, np.int32),
               allocs=torch.from_numpy(aa).to(dev))
    slots = medusa.materialize(**inp)
    # copy-free buffer contents (§4.3): classify, and dump the permanent buffers
    # offline
    plan = medusa.buffers_plan(inp["allocs"], t(capture_t, np.int32), slots.slot, slots.n_slots)
    buf_blob, rep_save = medusa.buffers_save(plan, t(allocs["base"], np.int64))
    torch.cuda.synchronize()
    cls = plan.cls.cpu().numpy()
    new_base = online_bases(A["L"], allocs, A["events"])
    live = allocs["t_free"] == T_END
    for i in np.nonzero(live)[0]:
        if cls[i] == medusa.BUF_PARAM or (cls[i] == medusa.BUF_UNUSED and not _in_capture(allocs, capture_t, i)):
            # allocated before the captures (weights, inputs, workspaces): "the online
            # process loads the same weights / inputs"
            _check(rt.cudaMemcpy(int(new_base[i]), int(allocs["base"][i]), int(allocs["size"][i]),
                                 rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice))
        else:  # the graphs' own pool: poisoned; only the permanent buffers come back (from the blob)
            _check(rt.cudaMemset(int(new_base[i]), 0xEE, int(allocs["size"][i])))
    for i in np.nonzero(live)[0]:  # nothing may still point into the first arena
        _check(rt.cudaMemset(int(allocs["base"][i]), 0xFF, int(allocs["size"][i])))
    torch.cuda.synchronize()
    dst, _, rep = medusa.restore(inp["words"], slots, t(allocs["base"], np.int64), t(new_base, np.int64),
                                 t(allocs["size"], np.int64))
    restored = medusa.to_numpy_u64(dst)
    report = medusa.report_numpy(rep)
    # the restored parameters into a clone of every graph (NEXT-2), run them all
    clones = [_check(cu.cuGraphClone(g)) for g in A["graphs"]]
    keep = []
    for k, r in enumerate(used):
        blob = restored[int(off[k]):int(off[k + 1])].tobytes()
        node_b = _check(cu.cuGraphNodeFindInClone(r["node"], clones[r["graph"]]))
        if r["kind"] == "kernel":
            hb = ctypes.create_string_buffer(blob, max(len(blob), 8))
            argv = (ctypes.c_void_p * max(len(r["layout"]), 1))()
            for i, (o, _s) in enumerate(r["layout"]):
                argv[i] = ctypes.addressof(hb) + o
            p = r["params"]
            p.kernelParams = ctypes.addressof(argv)
            p.extra = 0
            _check(cu.cuGraphKernelNodeSetParams(node_b, p))
            keep += [hb, argv]
        else:
            p = r["params"]
            p.dst = int.from_bytes(blob, "little")
            _check(cu.cuGraphMemsetNodeSetParams(node_b, p))
    stream = torch.cuda.current_stream().cuda_stream
    execs = [_check(cu.cuGraphInstantiate(gb, 0)) for gb in clones]

    def run_and_read():
        for ge in execs:
            _check(cu.cuGraphLaunch(ge, stream))
        torch.cuda.synchronize()
        # the outputs: each of A's output tensors sits in some traced allocation; same offset in B
        res = []
        for out, ref in zip(A["outs"], A["refs"]):
            op = out.data_ptr()
            i = int(np.nonzero((allocs["base"] <= op) & (op < allocs["base"] + allocs["size"]))[0][-1])
            ob = torch.empty_like(ref)
            _check(rt.cudaMemcpy(ob.data_ptr(), int(new_base[i]) + (op - int(allocs["base"][i])),
                                 ob.numel() * ob.element_size(), rt.cudaMemcpyKind.cudaMemcpyDeviceToHost))
            res.append(ob)
        return res

    # negative control: the permanent buffers not restored yet (poisoned)
    outs_unrestored = run_and_read()
    rep_buf = medusa.buffers_restore(plan, buf_blob, t(new_base, np.int64), t(allocs["size"], np.int64))
    torch.cuda.synchronize()
    outs_b = run_and_read()
    n_kernel = sum(1 for r in recs if r["kind"] == "kernel")
    names = set()
    for r in used:
        if r["kind"] == "kernel":
            res = cu.cuKernelGetName(r["params"].kern) if int(r["params"].kern) else cu.cuFuncGetName(r["params"].func)
            if int(res[0]) == 0:
                names.add(res[1].decode() if isinstance(res[1], bytes) else str(res[1]))
    n_pre = int(np.sum(allocs["t_alloc"] < int(capture_t[0, 0]))) if capture_t.size else len(allocs)
    return dict(words=words, off=off, node_t=node_t, allocs=allocs, slots=slots, new_base=new_base, n_pre=n_pre,
                restored=restored, report=report, refs=A["refs"], outs_b=outs_b, n_graphs=len(A["graphs"]),
                capture_t=capture_t, buf_class=cls, n_perm=plan.n_perm, blob_bytes=plan.blob_bytes,
                perm=plan.perm.cpu().numpy().view(np.uint32).copy(), perm_off=plan.perm_off.cpu().numpy().copy(),
                buf_report=[int(x) for x in medusa.report_numpy(rep_save)] + [int(x) for x in medusa.report_numpy(rep_buf)],
                outs_unrestored=outs_unrestored, magic_allocs=[_alloc_of(allocs, m.data_ptr()) for m in A["magic"]],
                n_nodes=len(recs),
                n_kernel=n_kernel, n_other=sum(1 for r in recs if r["kind"] == "other"), kernel_names=names)


# ---------------------------------------------------------------------------
# Offline / online in separate processes (NEXT-4: kernel addresses in a fresh
# process come from a triggering capture + module / library enumeration)

_ATTRS = ("CU_LAUNCH_ATTRIBUTE_CLUSTER_DIMENSION", "CU_LAUNCH_ATTRIBUTE_CLUSTER_SCHEDULING_POLICY_PREFERENCE",
          "CU_LAUNCH_ATTRIBUTE_PRIORITY")


def _kernel_name(cu, p):
    res = cu.cuKernelGetName(p.kern) if int(p.kern) else cu.cuFuncGetName(p.func)
    if int(res[0]) != 0:
        return None
    return res[1].decode() if isinstance(res[1], bytes) else str(res[1])


def _node_attrs(cu, node):
    out = {}
    for a in _ATTRS:
        aid = getattr(cu.CUkernelNodeAttrID, a)
        r = cu.cuGraphKernelNodeGetAttribute(node, aid)
        if int(r[0]) != 0:
            continue
        v = r[1]
        if a.endswith("CLUSTER_DIMENSION"):
            out[a] = [int(v.clusterDim.x), int(v.clusterDim.y), int(v.clusterDim.z)]
        elif a.endswith("POLICY_PREFERENCE"):
            out[a] = int(v.clusterSchedulingPolicyPreference)
        else:
            out[a] = int(v.priority)
    return out


def offline(torch, medusa, out_dir, seed=0):
    """The offline (materialization-time) process: capture, extract, materialize on
    the GPU; save everything the online process needs (the indirect index
    pointer table, kernel-name ids, launch configurations, the trace)."""
    import json
    from cuda.bindings import driver as cu

    A = capture(torch, seed=seed)
    recs = parameter_image(cu, A["nodes"])
    words, off, node_t, allocs, used, capture_t = trace_arrays(A["events"], recs)
    if any(r["kind"] != "kernel" for r in used):
        raise RuntimeError("offline/online demo handles kernel nodes only")
    dev = torch.device("cuda")
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(dev)
    aa = np.ascontiguousarray(allocs).view(np.int64).reshape(-1, 3)
    d_allocs = torch.from_numpy(aa).to(dev)
    slots = medusa.materialize(t(words, np.int64), t(off, np.int64), t(node_t, np.int32), d_allocs)
    # the permanent buffers' contents (§4.3): classified and dumped offline
    plan = medusa.buffers_plan(d_allocs, t(capture_t, np.int32), slots.slot, slots.n_slots)
    blob, rep_save = medusa.buffers_save(plan, t(allocs["base"], np.int64))
    torch.cuda.synchronize()
    if int(medusa.report_numpy(rep_save)[0]):
        raise RuntimeError("medusa_buffers_save reported segments it could not copy")
    names, func_id, meta = [], [], []
    for r in used:
        nm = _kernel_name(cu, r["params"])
        if nm not in names:
            names.append(nm)
        func_id.append(names.index(nm))
        p = r["params"]
        meta.append(dict(graph=r["graph"], grid=[int(p.gridDimX), int(p.gridDimY), int(p.gridDimZ)],
                         block=[int(p.blockDimX), int(p.blockDimY), int(p.blockDimZ)], smem=int(p.sharedMemBytes),
                         layout=r["layout"], attrs=_node_attrs(cu, r["node"])))
    outs = []
    for o, ref in zip(A["outs"], A["refs"]):
        op = o.data_ptr()
        i = int(np.nonzero((allocs["base"] <= op) & (op < allocs["base"] + allocs["size"]))[0][-1])
        outs.append(dict(alloc=i, offset=op - int(allocs["base"][i]), shape=list(ref.shape)))
        np.save(os.path.join(out_dir, f"ref{len(outs) - 1}.npy"), ref.numpy())
    first_capture = int(np.nonzero(A["events"][:, 0] == 3)[0][0])
    np.savez(os.path.join(out_dir, "image.npz"), words=words, off=off, node_t=node_t, allocs=aa,
             mask=slots.mask.cpu().numpy(), chunk_base=slots.chunk_base.cpu().numpy(),
             slot=slots.slot[: slots.n_slots].cpu().numpy(), func_id=np.array(func_id, np.uint32),
             events=A["events"], buf_perm=plan.perm.cpu().numpy(), buf_perm_off=plan.perm_off.cpu().numpy(),
             buf_blob=blob[: plan.blob_bytes].cpu().numpy())
    json.dump(dict(names=names, meta=meta, outs=outs, n_slots=slots.n_slots, graphs=len(A["graphs"]),
                   load_events=first_capture, seed=seed, n_perm=plan.n_perm, blob_bytes=plan.blob_bytes),
              open(os.path.join(out_dir, "meta.json"), "w"))
    return dict(nodes=len(used), names=len(names), slots=slots.n_slots, n_perm=plan.n_perm,
                blob_bytes=plan.blob_bytes)


def _dlsym_kernels(torch, names):
    """dlopen the library, dlsym the kernel's (host stub) symbol, then
    cudaGetFuncBySymbol.  Returns {name: CUfunction}."""
    # the CUDA runtime instance PyTorch registered its kernels with
    cudart = None
    for soname in ("libcudart.so.12", "libcudart.so"):
        try:
            cudart = ctypes.CDLL(soname, mode=os.RTLD_NOLOAD | os.RTLD_GLOBAL)
            break
        except OSError:
            continue
    if cudart is None:
        return {}
    cudart.cudaGetFuncBySymbol.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.c_void_p]
    cudart.cudaGetFuncBySymbol.restype = ctypes.c_int

    libdir = os.path.join(os.path.dirname(torch.__file__), "lib")
    libs = []
    for f in ("libtorch_cuda.so", "libc10_cuda.so"):
        try:
            libs.append(ctypes.CDLL(os.path.join(libdir, f), mode=os.RTLD_NOLOAD | os.RTLD_GLOBAL))
        except OSError:
            pass
    out = {}
    for nm in names:
        for lib in libs:
            try:
                stub = ctypes.cast(getattr(lib, nm), ctypes.c_void_p).value
            except AttributeError:
                continue
            fn = ctypes.c_void_p(0)
            if cudart.cudaGetFuncBySymbol(ctypes.byref(fn), ctypes.c_void_p(stub)) == 0 and fn.value:
                out[nm] = int(fn.value)
                break
    return out


def _resolve_kernels(torch, cu, model, ids, mask, names):
    """Kernel addresses in this process (§5): dlsym + cudaGetFuncBySymbol first;
    for the rest, capture the model's first layer (the triggering kernels,
    P:254-259), take the addresses of its nodes, and enumerate the modules /
    libraries those kernels came from, matching names.
    Returns ({name: CUfunction}, stats)."""
    found = _dlsym_kernels(torch, names)
    n_dlsym = len(found)
    g = torch.cuda.CUDAGraph(keep_graph=True)
    with torch.no_grad(), torch.cuda.graph(g):  # default pool: not part of the replayed trace
        model.layers[0](model.emb(ids[:1]), mask)  # the first layer
    graph = cu.CUgraph(g.raw_cuda_graph())
    n = int(cu.cuGraphGetNodes(graph, 0)[2])
    modules, libraries = {}, {}
    n_trig = 0
    for node in cu.cuGraphGetNodes(graph, n)[1]:
        if cu.cuGraphNodeGetType(node)[1] != cu.CUgraphNodeType.CU_GRAPH_NODE_TYPE_KERNEL:
            continue
        p = cu.cuGraphKernelNodeGetParams(node)[1]
        nm = _kernel_name(cu, p)
        if int(p.kern):
            fn = _check(cu.cuKernelGetFunction(p.kern))
            lib = _check(cu.cuKernelGetLibrary(p.kern))
            libraries[int(lib)] = lib
        else:
            fn = p.func
            mod = _check(cu.cuFuncGetModule(fn))
            modules[int(mod)] = mod
        if nm in names and nm not in found:
            found[nm] = int(fn)
            n_trig += 1
    n_enum = 0
    for mod in modules.values():
        cnt = _check(cu.cuModuleGetFunctionCount(mod))
        for fn in _check(cu.cuModuleEnumerateFunctions(cnt, mod)):
            r = cu.cuFuncGetName(fn)
            nm = (r[1].decode() if isinstance(r[1], bytes) else str(r[1])) if int(r[0]) == 0 else None
            if nm in names and nm not in found:
                found[nm] = int(fn)
                n_enum += 1
    for lib in libraries.values():
        cnt = _check(cu.cuLibraryGetKernelCount(lib))
        for k in _check(cu.cuLibraryEnumerateKernels(cnt, lib)):
            r = cu.cuKernelGetName(k)
            nm = (r[1].decode() if isinstance(r[1], bytes) else str(r[1])) if int(r[0]) == 0 else None
            if nm in names and nm not in found:
                found[nm] = int(_check(cu.cuKernelGetFunction(k)))
                n_enum += 1
    stats = dict(dlsym=n_dlsym, triggering=n_trig, enumerated=n_enum,
                 unresolved=sum(1 for nm in names if nm not in found))
    return found, stats


def online(torch, medusa, in_dir, arena_bytes=1 << 30):
    """The online process (a fresh one): load the same model into the traced
    pool, replay the rest of the offline allocation sequence, resolve kernel
    addresses, restore (relocate + validate + kernel-address fill), build every
    graph from scratch and run it.  Returns the facts to check."""
    import json
    from cuda.bindings import driver as cu
    from cuda.bindings import runtime as rt

    meta = json.load(open(os.path.join(in_dir, "meta.json")))
    z = np.load(os.path.join(in_dir, "image.npz"))
    ev_a = z["events"]
    L = _lib()
    if L.ta_init(arena_bytes) != 0:
        raise RuntimeError("tracing allocator: cudaMalloc of the arenas failed")
    alloc = torch.cuda.memory.CUDAPluggableAllocator(build(), "ta_malloc", "ta_free")
    # the second arena: a fresh process on the same box may receive the very same
    # virtual addresses for its first cudaMalloc as the offline process did, so the
    # first arena would hand out the offline addresses again (nothing to relocate);
    # the second one lies elsewhere by construction
    L.ta_select(1)
    L.ta_clear()
    L.ta_log(1)
    pool = torch.cuda.MemPool(alloc.allocator())
    torch.manual_seed(meta["seed"])
    batches = (8, 4, 2, 1)
    with torch.cuda.use_mem_pool(pool):  # the same loading sequence as offline
        model = tiny_decoder(torch).cuda().eval()
        seq = meta["outs"][0]["shape"][1]
        ids = torch.randint(0, 512, (max(batches), seq), device="cuda")
        mask = torch.full((seq, seq), float("-inf"), device="cuda").triu(1)
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s), torch.no_grad():
            for b in batches:
                model(ids[:b], mask)
        torch.cuda.current_stream().wait_stream(s)
        torch.cuda.synchronize()
    L.ta_log(0)
    n_ev = L.ta_events(None, 0)
    buf = (ctypes.c_int64 * (5 * n_ev))()
    L.ta_events(buf, n_ev)
    ev_b = np.frombuffer(buf, dtype=np.int64).reshape(n_ev, 5)
    nl = meta["load_events"]
    same_loading = n_ev == nl and bool(np.array_equal(ev_b[:, [0, 2]], ev_a[:nl, [0, 2]]))
    # new base of every allocation ordinal: loading phase as it happened here, the
    # rest replayed
    L.ta_free.argtypes = [ctypes.c_void_p, ctypes.c_ssize_t, ctypes.c_int, ctypes.c_void_p]
    new_base = []
    moved = {}
    for k in range(ev_a.shape[0]):
        kind, ptr = int(ev_a[k, 0]), int(ev_a[k, 1]) & ((1 << 64) - 1)
        if kind == 1:
            nb = int(ev_b[k, 1]) & ((1 << 64) - 1) if k < nl else L.ta_raw_malloc(int(ev_a[k, 2]))
            new_base.append(nb)
            moved[ptr] = nb
        elif kind == 2 and k >= nl and ptr in moved:
            L.ta_free(ctypes.c_void_p(moved.pop(ptr)), 0, 0, None)
    new_base = np.array(new_base, np.uint64)
    allocs = z["allocs"].view(np.uint64).reshape(-1, 3)
    # kernel addresses
    found, kstats = _resolve_kernels(torch, cu, model, ids, mask, meta["names"])
    table = np.array([found.get(nm, 0) for nm in meta["names"]], np.uint64)
    dev = torch.device("cuda")
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a).view(dt)).to(dev)
    slots = medusa.Slots(t(z["mask"], np.int32), t(z["chunk_base"], np.int32), t(z["slot"], np.int64),
                         int(meta["n_slots"]))
    medusa.kernel_table_set(t(table, np.int64))
    dst, fout, rep = medusa.restore(t(z["words"], np.int64), slots, t(allocs[:, 0], np.int64),
                                    t(new_base, np.int64), t(allocs[:, 1], np.int64), t(z["func_id"], np.int32))
    # the permanent buffers' saved contents into the replayed allocations (§4.3)
    blob = torch.from_numpy(z["buf_blob"]).to(dev)
    if blob.numel() < 16:
        blob = torch.zeros(16, dtype=torch.uint8, device=dev)
    bplan = medusa.BufferPlan(None, t(z["buf_perm"], np.int32), t(z["buf_perm_off"], np.int64), int(meta["n_perm"]),
                              int(meta["blob_bytes"]))
    rep_buf = medusa.buffers_restore(bplan, blob, t(new_base, np.int64), t(allocs[:, 1], np.int64))
    torch.cuda.synchronize()
    restored = medusa.to_numpy_u64(dst)
    func_out = medusa.to_numpy_u64(fout)
    report = medusa.report_numpy(rep)
    buf_report = [int(x) for x in medusa.report_numpy(rep_buf)]
    if kstats["unresolved"] or int(report[5]):
        missing = [nm for nm in meta["names"] if nm not in found]
        return dict(same_loading=same_loading, kernels=kstats, report=[int(x) for x in report],
                    unresolved_names=missing[:5], outputs_equal=[])
    # every graph built from scratch: nodes in launch order, one chain
    off = z["off"]
    keep, graphs = [], [_check(cu.cuGraphCreate(0)) for _ in range(meta["graphs"])]
    prev = [None] * meta["graphs"]
    for j, m in enumerate(meta["meta"]):
        blob = restored[int(off[j]):int(off[j + 1])].tobytes()
        hb = ctypes.create_string_buffer(blob, max(len(blob), 8))
        argv = (ctypes.c_void_p * max(len(m["layout"]), 1))()
        for i, (o, _s) in enumerate(m["layout"]):
            argv[i] = ctypes.addressof(hb) + o
        keep += [hb, argv]
        p = cu.CUDA_KERNEL_NODE_PARAMS()
        p.func = cu.CUfunction(int(func_out[j]))
        p.gridDimX, p.gridDimY, p.gridDimZ = m["grid"]
        p.blockDimX, p.blockDimY, p.blockDimZ = m["block"]
        p.sharedMemBytes = m["smem"]
        p.kernelParams = ctypes.addressof(argv)
        p.extra = 0
        gi = m["graph"]
        deps = [prev[gi]] if prev[gi] is not None else []
        node = _check(cu.cuGraphAddKernelNode(graphs[gi], deps, len(deps), p))
        for a, v in m["attrs"].items():
            val = cu.CUkernelNodeAttrValue()
            if a.endswith("CLUSTER_DIMENSION"):
                val.clusterDim.x, val.clusterDim.y, val.clusterDim.z = v
            elif a.endswith("POLICY_PREFERENCE"):
                val.clusterSchedulingPolicyPreference = v
            else:
                val.priority = v
            _check(cu.cuGraphKernelNodeSetAttribute(node, getattr(cu.CUkernelNodeAttrID, a), val))
        prev[gi] = node
    stream = torch.cuda.current_stream().cuda_stream
    for g in graphs:
        _check(cu.cuGraphLaunch(_check(cu.cuGraphInstantiate(g, 0)), stream))
    torch.cuda.synchronize()
    equal = []
    for k, o in enumerate(meta["outs"]):
        ref = np.load(os.path.join(in_dir, f"ref{k}.npy"))
        ob = np.empty_like(ref)
        _check(rt.cudaMemcpy(ob.ctypes.data, int(new_base[o["alloc"]]) + o["offset"], ob.nbytes,
                             rt.cudaMemcpyKind.cudaMemcpyDeviceToHost))
        equal.append(bool(np.array_equal(ob, ref)))
    moved_bases = int(np.sum(new_base != allocs[:, 0]))
    return dict(same_loading=same_loading, kernels=kstats, report=[int(x) for x in report], outputs_equal=equal,
                nodes=len(meta["meta"]), allocations=int(len(new_base)), moved_bases=moved_bases,
                slots=int(meta["n_slots"]), n_perm=int(meta["n_perm"]), blob_bytes=int(meta["blob_bytes"]),
                buf_report=buf_report)
