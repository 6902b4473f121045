"""Seeded synthetic CUDA-graph sets shaped like the paper's workloads.

Input generator shared by the oracle tests and the CUDA path (it holds none of
the method's arithmetic: every pointer word is *constructed* from an
allocation the simulated allocator handed out, never classified).

What it reproduces (a [model] fixed for reproducibility):
  * Table 1: the exact per-model node totals over 35
    capture batch sizes, as 35 graphs of 2 + L*k_b nodes;
  * vLLM's loading order: weights -> profiling
    forward (KV-cache sizing) -> KV cache -> static capture inputs ->
    for every batch size, largest first and one at a time: warm-up
    forward then the captured forward;
  * a caching allocator with block reuse (Fig. 6);
  * two 4-byte permanent buffers per tagged (qkv GEMM) kernel, never freed
    (9.0% of kernels);
  * kernel names per node; GEMM names are "trigger" (hidden
    from dlsym), the rest "dlsym";
  * every 8-byte word of every node's parameter image tagged with what it is
    (pointer / constant / gap / one-past-end / dangling / deliberate false
    positive), so tests can pin the oracle against construction (pins P8, P11);
  * online replay addresses: every allocator segment moved to a
    new, disjoint VA region in shuffled order -> the relocation is not a
    constant shift; sizes are unchanged ("identical control flow").
Event positions are one total order over ALLOC / FREE / LAUNCH.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

from .allocator import CachingAllocator, LiveSet, MiB

# ---- tags ------------------------------------------------------------------
TAG_CONST = 0  # plain constant (dims, strides, fp32 bit patterns, nulls)
TAG_PTR = 1  # data pointer into an allocation live at launch (truth id/off)
TAG_GAP = 2  # high-prefix word inside a never-allocated VA hole
TAG_OPE = 3  # one-past-end of a live allocation (truth id = block starting there, else -1)
TAG_DANGLING = 4  # inside an allocation that was freed before the launch
TAG_FP = 5  # constant that deliberately aliases a live allocation
TAG_NAMES = ["const", "ptr", "gap", "one_past_end", "dangling", "false_positive"]

T_NEVER = 0xFFFFFFFF
ALLOC_DTYPE = np.dtype([("base", "<u8"), ("size", "<u8"), ("t_alloc", "<u4"), ("t_free", "<u4")])
assert ALLOC_DTYPE.itemsize == 24

OLD_REGION = 0x7F00_0000_0000  # model m lives at OLD_REGION + m * 2**40 (high prefix)
NEW_REGION = 0xC000_0000_0000  # replayed (online) addresses, disjoint from every old region
REGION = 1 << 40
N_REGIONS = 16
OLD_BAND = (OLD_REGION, OLD_REGION + N_REGIONS * REGION)
NEW_BAND = (NEW_REGION, NEW_REGION + N_REGIONS * REGION)

# Adversarial rates, as a share of constant words.
_RATES = (0.01, 0.005, 0.002, 0.0005)  # gap, one-past-end, dangling, deliberate FP
# Pointer offsets: 70% base, 25% 16-B aligned interior, 5% 2-B aligned interior.
P_INTERIOR16, P_INTERIOR2 = 0.25, 0.05

# vLLM 0.4 _BATCH_SIZES_TO_CAPTURE [ext]; the paper: "35 different batch sizes".
BATCH_SIZES = [1, 2, 4] + [8 * i for i in range(1, 33)]
assert len(BATCH_SIZES) == 35


@dataclasses.dataclass(frozen=True)
class ModelCfg:
    name: str
    L: int
    H: int
    I: int
    heads: int
    kv_heads: int
    vocab: int
    param_gb: float
    ksplit: tuple  # ((count, k), (count, k+1)) over the 35 graphs, small batch sizes first
    qwen: bool = False


# L/H/I/heads from the HF configs [ext]; parameter sizes and node totals: Table 1.
MODELS = {
    m.name: m
    for m in [
        ModelCfg("falcon-7b", 32, 4544, 18176, 71, 1, 65024, 13.4, ((7, 12), (28, 13))),
        ModelCfg("llama2-7b", 32, 4096, 11008, 32, 32, 32000, 12.6, ((31, 11), (4, 12))),
        ModelCfg("llama2-13b", 40, 5120, 13824, 40, 40, 32000, 24.2, ((18, 11), (17, 12))),
        ModelCfg("qwen1.5-0.5b", 24, 1024, 2816, 16, 16, 151936, 1.2, ((8, 10), (27, 11)), True),
        ModelCfg("qwen1.5-1.8b", 24, 2048, 5504, 16, 16, 151936, 3.4, ((25, 11), (10, 12)), True),
        ModelCfg("qwen1.5-4b", 40, 2560, 6912, 20, 20, 151936, 7.4, ((18, 11), (17, 12)), True),
        ModelCfg("qwen1.5-7b", 32, 4096, 11008, 32, 32, 151936, 14.4, ((19, 11), (16, 12)), True),
        ModelCfg("qwen1.5-14b", 40, 5120, 13696, 40, 40, 152064, 26.4, ((13, 11), (22, 12)), True),
        ModelCfg("yi-6b", 32, 4096, 11008, 32, 4, 64000, 11.3, ((19, 11), (16, 12))),
        ModelCfg("yi-9b", 48, 4096, 11008, 32, 4, 64000, 16.4, ((19, 11), (16, 12))),
    ]
}
ALL10 = list(MODELS)
TABLE1_NODES = {
    "falcon-7b": 14406, "llama2-7b": 12518, "llama2-13b": 16150, "qwen1.5-0.5b": 9118,
    "qwen1.5-1.8b": 9550, "qwen1.5-4b": 16150, "qwen1.5-7b": 12902, "qwen1.5-14b": 16350,
    "yi-6b": 12902, "yi-9b": 19318,
}  # P:249; sum 139,364

# Kernel-node parameter images: (words, pointer word positions).  Byte sizes are
# SURVEY.md Appendix A's; the layouts are a [model] of cuFuncGetParamInfo offsets.
TEMPLATES = {
    "embed": (84, (0, 28, 56)),  # index_select, 3 TensorInfo structs by value (672 B)
    "rmsnorm": (5, (0, 1, 2)),  # 40 B
    "fused_add_rmsnorm": (5, (0, 1, 2)),  # 40 B
    "gemm": (48, (0, 1, 2, 3)),  # 384 B; + bias at 4 (Qwen qkv), permanent buffers at 20, 21
    "rotary": (9, (0, 1, 2, 3)),  # 72 B
    "reshape_and_cache": (10, (0, 1, 2, 3, 4)),  # 80 B
    "paged_attention_v1": (13, (0, 1, 2, 3, 4, 5)),  # 104 B
    "silu_and_mul": (3, (0, 1)),  # 24 B
    "splitk_reduce": (8, (0, 1, 2)),  # 64 B
    "pa_v2_reduce": (12, (0, 1, 2, 3, 4)),  # 96 B
    "elementwise": (56, (0, 19, 38)),  # 448 B
}
GEMM_BIAS_POS = 4
GEMM_PERM_POS = (20, 21)
DLSYM, TRIGGER = 0, 1


def _gemm_bucket(b: int) -> int:
    for i, hi in enumerate((4, 16, 48, 96, 176)):
        if b <= hi:
            return i
    return 5


@dataclasses.dataclass
class GraphSet:
    """One materialization input (+ the online replay and ground truth)."""

    name: str
    words: np.ndarray  # u64[n_words] concatenated, 8-B zero-padded parameter images
    node_word_off: np.ndarray  # u64[N+1] CSR
    node_t: np.ndarray  # u32[N] launch event position (strictly increasing)
    func_id: np.ndarray  # u32[N] kernel-name id
    allocs: np.ndarray  # ALLOC_DTYPE[n_alloc], index = allocation ordinal
    new_base: np.ndarray  # u64[n_alloc] replayed addresses
    new_size: np.ndarray  # u64[n_alloc]
    table: np.ndarray  # u64[K] kernel addresses resolved online
    func_kind: np.ndarray  # u8[K] DLSYM / TRIGGER
    tags: np.ndarray  # u8[n_words]
    truth_id: np.ndarray  # i64[n_words] (-1 = none)
    truth_off: np.ndarray  # u64[n_words]
    node_model: np.ndarray  # u16[N]
    node_bs: np.ndarray  # u16[N]
    node_perm: np.ndarray  # bool[N] kernel owns permanent buffers
    alloc_kind: np.ndarray  # u8[n_alloc]: 0 weight 1 kv 2 static 3 profiling 4 warmup 5 capture-temp 6 permanent
    models: list
    capture_t: np.ndarray = None  # u32[n_graphs, 2]: event positions (begin, end) of each graph's capture

    @property
    def n_words(self):
        return int(self.words.size)

    @property
    def n_nodes(self):
        return int(self.node_t.size)

    @property
    def n_alloc(self):
        return int(self.allocs.size)


AK_WEIGHT, AK_KV, AK_STATIC, AK_PROFILE, AK_WARMUP, AK_CAPTURE, AK_PERM = range(7)


class _Builder:
    def __init__(self, seed: int, rates=_RATES):
        self.rng = np.random.default_rng(seed)
        self.rates = rates
        self.t = 0
        self.a_base, self.a_size, self.a_ta, self.a_tf = [], [], [], []
        self.a_seg, self.a_kind = [], []
        self.seg_model, self.seg_base, self.seg_size = [], [], []
        self.blobs, self.btags, self.btid, self.btoff = [], [], [], []
        self.n_t, self.n_fid, self.n_model, self.n_bs, self.n_perm = [], [], [], [], []
        self.func_names = {}
        self.func_kind = []
        self.models = []
        self.captures = []
        self._const_cache = {}
        self.rate_scale = 1.0  # the toy set uses 4x rates so every category shows up

    # -- per-model state ---------------------------------------------------
    def begin_model(self, m_index: int, cfg):
        self.m = m_index
        self.cfg = cfg
        self.alloc = CachingAllocator(OLD_REGION + m_index * REGION, self.rng)
        self.seg_off = len(self.seg_base)
        self.live = LiveSet()
        self.recent_freed = []
        self.models.append(cfg.name if hasattr(cfg, "name") else str(cfg))

    def end_model(self):
        for s in self.alloc.segments:
            self.seg_model.append(self.m)
            self.seg_base.append(s.base)
            self.seg_size.append(s.size)
        self.model_gaps = getattr(self, "model_gaps", [])

    # -- trace events --------------------------------------------------------
    def malloc(self, nbytes, kind, pool="default"):
        addr, size, seg = self.alloc.malloc(nbytes, pool)
        self.t += 1
        aid = len(self.a_base)
        self.a_base.append(addr)
        self.a_size.append(size)
        self.a_ta.append(self.t)
        self.a_tf.append(T_NEVER)
        self.a_seg.append(self.seg_off + seg.index)
        self.a_kind.append(kind)
        self.live.add(addr, size, aid)
        return aid

    def free(self, aid):
        self.alloc.free(self.a_base[aid])
        self.t += 1
        self.a_tf[aid] = self.t
        self.live.remove(self.a_base[aid], aid)
        self.recent_freed.append(aid)
        if len(self.recent_freed) > 512:
            del self.recent_freed[:256]

    def begin_capture(self):
        """cudaStreamBeginCapture: an event of its own in the one total order."""
        self.t += 1
        self._capture_begin = self.t

    def end_capture(self):
        self.t += 1
        self.captures.append((self._capture_begin, self.t))

    # -- nodes ---------------------------------------------------------------
    def func(self, key, kind):
        fid = self.func_names.get(key)
        if fid is None:
            fid = len(self.func_kind)
            self.func_names[key] = fid
            self.func_kind.append(kind)
        return fid

    def _consts(self, tmpl, b, n_words):
        key = (self.m, tmpl, b)
        c = self._const_cache.get(key)
        if c is None:
            cfg = self.cfg
            H, I, heads = cfg.H, cfg.I, cfg.heads
            hd = H // heads
            vals = np.zeros(n_words, dtype=np.uint64)
            f32 = lambda x: int(np.float32(x).view(np.uint32))
            choices = [
                (b << 32) | H,  # packed (tokens, hidden)
                H * 2,  # row stride in bytes
                (f32(0.0) << 32) | f32(1.0),  # alpha / beta
                0,  # null pointer / flags
                (heads << 32) | hd,
                f32(1e-6) | (H << 32),  # eps | hidden
                (2 * I << 32) | I,
                0xFFFFFFFFFFFFFFFF,  # -1 (e.g. ignore index)
                f32(1.0 / math.sqrt(hd)),
                (cfg.vocab << 32) | 16,
                b * H,
                7,
            ]
            for p in range(n_words):
                vals[p] = np.uint64(choices[(p * 7 + len(tmpl)) % len(choices)])
            c = vals
            self._const_cache[key] = c
        return c

    def node(self, tmpl, ptrs, fkey, fkind, b, perms=(), bias=None):
        """Record one captured kernel launch.  ptrs: list of (aid, offset)."""
        n_words, ppos = TEMPLATES[tmpl]
        vals = self._consts(tmpl, b, n_words).copy()
        tags = np.zeros(n_words, dtype=np.uint8)
        tid = np.full(n_words, -1, dtype=np.int64)
        toff = np.zeros(n_words, dtype=np.uint64)
        self.t += 1
        rng = self.rng
        slots = list(zip(ppos, ptrs))
        if bias is not None:
            slots.append((GEMM_BIAS_POS, bias))
        for pos, pa in zip(GEMM_PERM_POS, perms):
            slots.append((pos, (pa, 0)))
        u = rng.random(len(slots))
        for (pos, (aid, off)), uu in zip(slots, u):
            size = self.a_size[aid]
            if off == 0 and uu < P_INTERIOR16 + P_INTERIOR2:
                if uu < P_INTERIOR16:
                    off = int(rng.integers(0, size // 16)) * 16
                else:
                    off = int(rng.integers(0, size // 2)) * 2
            vals[pos] = self.a_base[aid] + off
            tags[pos] = TAG_PTR
            tid[pos] = aid
            toff[pos] = off
        self._adversarial(vals, tags, tid, toff)
        self.blobs.append(vals)
        self.btags.append(tags)
        self.btid.append(tid)
        self.btoff.append(toff)
        self.n_t.append(self.t)
        self.n_fid.append(self.func(fkey, fkind))
        self.n_model.append(self.m)
        self.n_bs.append(b)
        self.n_perm.append(len(perms) > 0)

    def _adversarial(self, vals, tags, tid, toff):
        rng = self.rng
        cidx = np.flatnonzero(tags == TAG_CONST)
        if cidx.size == 0:
            return
        # Plain constants never enter the old or new address bands: constants that
        # alias memory are placed on purpose below and tagged (pins P7, P8, P11).
        cv = vals[cidx]
        bad = ((cv >= OLD_BAND[0]) & (cv < OLD_BAND[1])) | ((cv >= NEW_BAND[0]) & (cv < NEW_BAND[1]))
        if bad.any():
            vals[cidx[bad]] ^= np.uint64(1 << 47)
        u = rng.random(cidx.size) / self.rate_scale
        RATE_GAP, RATE_OPE, RATE_DANGLING, RATE_FP = self.rates
        for p, uu in zip(cidx, u):
            if uu >= RATE_GAP + RATE_OPE + RATE_DANGLING + RATE_FP:
                continue
            if uu < RATE_GAP:
                lo, hi = self.alloc.gaps[int(rng.integers(0, len(self.alloc.gaps)))]
                vals[p] = lo + int(rng.integers(0, (hi - lo) // 8)) * 8
                tags[p] = TAG_GAP
            elif uu < RATE_GAP + RATE_OPE:
                aid = self.live.random_id(rng)
                if aid < 0:
                    continue
                w = self.a_base[aid] + self.a_size[aid]
                vals[p] = w
                tags[p] = TAG_OPE
                adj = self.live.starting_at(w)
                tid[p] = adj
                toff[p] = 0
            elif uu < RATE_GAP + RATE_OPE + RATE_DANGLING:
                if not self.recent_freed:
                    continue
                for _ in range(8):
                    aid = self.recent_freed[int(rng.integers(0, len(self.recent_freed)))]
                    w = self.a_base[aid] + int(rng.integers(0, self.a_size[aid] // 8)) * 8
                    if self.live.covering(w) < 0:
                        vals[p] = w
                        tags[p] = TAG_DANGLING
                        break
            else:
                aid = self.live.random_id(rng)
                if aid < 0:
                    continue
                off = int(rng.integers(0, self.a_size[aid] // 8)) * 8
                vals[p] = self.a_base[aid] + off
                tags[p] = TAG_FP
                tid[p] = aid
                toff[p] = off

    # -- finish --------------------------------------------------------------
    def build(self, name) -> GraphSet:
        rng = self.rng
        n_alloc = len(self.a_base)
        allocs = np.zeros(n_alloc, dtype=ALLOC_DTYPE)
        allocs["base"] = np.asarray(self.a_base, dtype=np.uint64)
        allocs["size"] = np.asarray(self.a_size, dtype=np.uint64)
        allocs["t_alloc"] = np.asarray(self.a_ta, dtype=np.uint32)
        allocs["t_free"] = np.asarray(self.a_tf, dtype=np.uint32)
        # Online replay: every segment lands somewhere else (shuffled, 2 MiB aligned).
        seg_base = np.asarray(self.seg_base, dtype=np.uint64)
        seg_new = np.zeros_like(seg_base)
        seg_model = np.asarray(self.seg_model)
        for m in np.unique(seg_model):
            idx = np.flatnonzero(seg_model == m)
            cur = NEW_REGION + int(m) * REGION
            for s in rng.permutation(idx):
                seg_new[s] = cur
                cur += self.seg_size[s] + 2 * MiB * int(rng.integers(0, 4))
        a_seg = np.asarray(self.a_seg, dtype=np.int64)
        new_base = seg_new[a_seg] + (allocs["base"] - seg_base[a_seg])
        n_off = np.zeros(len(self.blobs) + 1, dtype=np.uint64)
        n_off[1:] = np.cumsum([b.size for b in self.blobs])
        K = len(self.func_kind)
        table = (rng.integers(1, 1 << 40, size=K, dtype=np.uint64) << np.uint64(4)) | np.uint64(0x7F00_0000_0000_0000)
        cat = lambda xs, dt: (np.concatenate(xs).astype(dt) if xs else np.zeros(0, dt))
        return GraphSet(
            name=name,
            words=cat(self.blobs, np.uint64),
            node_word_off=n_off,
            node_t=np.asarray(self.n_t, dtype=np.uint32),
            func_id=np.asarray(self.n_fid, dtype=np.uint32),
            allocs=allocs,
            new_base=new_base.astype(np.uint64),
            new_size=allocs["size"].copy(),
            table=table.astype(np.uint64),
            func_kind=np.asarray(self.func_kind, dtype=np.uint8),
            tags=cat(self.btags, np.uint8),
            truth_id=cat(self.btid, np.int64),
            truth_off=cat(self.btoff, np.uint64),
            node_model=np.asarray(self.n_model, dtype=np.uint16),
            node_bs=np.asarray(self.n_bs, dtype=np.uint16),
            node_perm=np.asarray(self.n_perm, dtype=bool),
            alloc_kind=np.asarray(self.a_kind, dtype=np.uint8),
            models=list(self.models),
            capture_t=np.asarray(self.captures, dtype=np.uint32).reshape(-1, 2),
        )


# ---------------------------------------------------------------------------
# vLLM-shaped model program
# ---------------------------------------------------------------------------
def _k_of_batch(cfg: ModelCfg) -> dict:
    (c0, k0), (c1, k1) = cfg.ksplit
    assert c0 + c1 == 35
    asc = sorted(BATCH_SIZES)
    return {b: (k0 if i < c0 else k1) for i, b in enumerate(asc)}


def _run_model(B: _Builder, m_index: int, cfg: ModelCfg):
    B.begin_model(m_index, cfg)
    L, H, I, heads = cfg.L, cfg.H, cfg.I, cfg.heads
    hd = H // heads
    kvH = cfg.kv_heads * hd
    qkv_n = H + 2 * kvH
    first_alloc = len(B.a_size)
    # 1. weights: 6L+3 (Qwen: 7L+3 with the qkv bias), never freed.
    W = {}
    W["embed"] = B.malloc(cfg.vocab * H * 2, AK_WEIGHT)
    W["final_norm"] = B.malloc(H * 2, AK_WEIGHT)
    W["cos_sin"] = B.malloc(4096 * hd * 4, AK_WEIGHT)
    layers = []
    for _ in range(L):
        lw = {
            "ln1": B.malloc(H * 2, AK_WEIGHT),
            "qkv": B.malloc(qkv_n * H * 2, AK_WEIGHT),
            "o": B.malloc(H * H * 2, AK_WEIGHT),
            "ln2": B.malloc(H * 2, AK_WEIGHT),
            "gate_up": B.malloc(2 * I * H * 2, AK_WEIGHT),
            "down": B.malloc(H * I * 2, AK_WEIGHT),
        }
        if cfg.qwen:
            lw["qkv_bias"] = B.malloc(qkv_n * 2, AK_WEIGHT)
        layers.append(lw)
    weight_bytes = sum(B.a_size[a] for a in range(first_alloc, len(B.a_size)))

    ctx = dict(cfg=cfg, W=W, layers=layers, hd=hd, kvH=kvH, qkv_n=qkv_n)
    # 2. profiling forward (KV-cache sizing): 7L+4 temps, all freed.
    _forward(B, ctx, b=4096, k=10, pool="default", kind=AK_PROFILE, record=False, extra=2)
    # 3. KV cache: L blocks, never freed (A100-40GB basis).
    kv_total = max(int(0.9 * 40e9) - weight_bytes - int(1e9), 256 * MiB * L)
    kv_layer = (kv_total // L) // (2 * MiB) * (2 * MiB)
    ctx["kv"] = [B.malloc(kv_layer, AK_KV) for _ in range(L)]
    # 4. static capture inputs + cuBLAS workspace: 6, never freed.
    ctx["S"] = {
        "ids": B.malloc(256 * 8, AK_STATIC),
        "pos": B.malloc(256 * 8, AK_STATIC),
        "slot": B.malloc(256 * 8, AK_STATIC),
        "bt": B.malloc(256 * 512 * 4, AK_STATIC),
        "sl": B.malloc(256 * 4, AK_STATIC),
        "ws": B.malloc(4 * MiB + 1024, AK_STATIC),
    }
    kmap = _k_of_batch(cfg)
    # 5. capture, largest batch size first, one graph at a time.
    for b in sorted(BATCH_SIZES, reverse=True):
        _forward(B, ctx, b=b, k=kmap[b], pool="default", kind=AK_WARMUP, record=False)
        B.begin_capture()
        _forward(B, ctx, b=b, k=kmap[b], pool="graph", kind=AK_CAPTURE, record=True)
        B.end_capture()
    B.end_model()


def _forward(B: _Builder, ctx, b, k, pool, kind, record, extra=0):
    cfg = ctx["cfg"]
    W, layers = ctx["W"], ctx["layers"]
    H, I, heads = cfg.H, cfg.I, cfg.heads
    kvH, qkv_n = ctx["kvH"], ctx["qkv_n"]
    S = ctx.get("S")
    kv = ctx.get("kv")
    mname = cfg.name
    bucket = _gemm_bucket(b)

    def node(tmpl, ptrs, fkey=None, fkind=DLSYM, perms=(), bias=None):
        if record:
            B.node(tmpl, ptrs, (mname,) + (fkey or (tmpl,)), fkind, b, perms, bias)

    E = B.malloc(b * H * 2, kind, pool)  # embedding output; residual stream of the forward
    if record:
        node("embed", [(E, 0), (S["ids"], 0), (W["embed"], 0)])
    x = E
    half = None
    for li, lw in enumerate(layers):
        ws = B.malloc(b * H * 4, kind, pool)
        node("fused_add_rmsnorm", [(x, 0), (E, 0), (lw["ln1"], 0)])
        qkv = B.malloc(b * qkv_n * 2, kind, pool)
        perms = ()
        if record:
            perms = (B.malloc(4, AK_PERM, pool), B.malloc(4, AK_PERM, pool))
        node("gemm", [(x, 0), (lw["qkv"], 0), (qkv, 0), (qkv, 0)], ("gemm_qkv", bucket), TRIGGER,
             perms=perms, bias=((lw["qkv_bias"], 0) if cfg.qwen else None))
        if x != E:
            B.free(x)
        if record:
            qb = b * H * 2
            kb = b * kvH * 2
            half = B.a_size[kv[li]] // 2 // 16 * 16
            node("rotary", [(S["pos"], 0), (qkv, 0), (qkv, qb), (W["cos_sin"], 0)])
            node("reshape_and_cache", [(qkv, qb), (qkv, qb + kb), (kv[li], 0), (kv[li], half), (S["slot"], 0)])
        attn = B.malloc(b * H * 2, kind, pool)
        if record:
            node("paged_attention_v1", [(attn, 0), (qkv, 0), (kv[li], 0), (kv[li], half), (S["bt"], 0), (S["sl"], 0)])
            if k >= 12:
                node("pa_v2_reduce", [(attn, 0), (ws, 0), (ws, b * heads * 4), (ws, 2 * b * heads * 4), (S["sl"], 0)])
        B.free(qkv)
        o = B.malloc(b * H * 2, kind, pool)
        node("gemm", [(attn, 0), (lw["o"], 0), (o, 0), (o, 0)], ("gemm_o", bucket), TRIGGER)
        if k >= 11 and record:
            node("splitk_reduce", [(o, 0), (ws, 0), (S["ws"], 0)])
        B.free(attn)
        node("fused_add_rmsnorm", [(o, 0), (E, 0), (lw["ln2"], 0)])
        gu = B.malloc(b * 2 * I * 2, kind, pool)
        node("gemm", [(o, 0), (lw["gate_up"], 0), (gu, 0), (gu, 0)], ("gemm_gate_up", bucket), TRIGGER)
        B.free(o)
        act = B.malloc(b * I * 2, kind, pool)
        node("silu_and_mul", [(act, 0), (gu, 0)])
        B.free(gu)
        down = B.malloc(b * H * 2, kind, pool)
        node("gemm", [(act, 0), (lw["down"], 0), (down, 0), (down, 0)], ("gemm_down", bucket), TRIGGER)
        B.free(act)
        if k >= 13:
            node("elementwise", [(down, 0), (down, 0), (E, 0)])
        B.free(ws)
        x = down
    F = B.malloc(b * H * 2, kind, pool)
    node("rmsnorm", [(F, 0), (x, 0), (W["final_norm"], 0)])
    B.free(x)
    for _ in range(extra):  # profiling run: logits + sampler scratch
        e = B.malloc(256 * cfg.vocab * 4, kind, pool)
        B.free(e)
    B.free(F)
    B.free(E)


# ---------------------------------------------------------------------------
# Toy config C1: one bs=1 graph of a 2-layer decoder, 200 nodes, 64 allocations.
# ---------------------------------------------------------------------------
TOY_CFG = ModelCfg("toy-2layer", 2, 256, 688, 4, 4, 1000, 0.0, ((35, 99), (0, 100)))
_TOY_POOL = ["rmsnorm", "fused_add_rmsnorm", "gemm", "rotary", "reshape_and_cache",
             "paged_attention_v1", "silu_and_mul", "splitk_reduce", "pa_v2_reduce", "elementwise"]


def _run_toy(B: _Builder):
    cfg = TOY_CFG
    B.begin_model(0, cfg)
    B.rate_scale = 4.0
    rng = B.rng
    H, I = cfg.H, cfg.I
    W = [B.malloc(cfg.vocab * H * 2, AK_WEIGHT), B.malloc(H * 2, AK_WEIGHT), B.malloc(1 << 16, AK_WEIGHT)]
    LW = [[B.malloc(s, AK_WEIGHT) for s in (H * 2, 3 * H * H * 2, H * H * 2, H * 2, 2 * I * H * 2, H * I * 2)]
          for _ in range(2)]
    KV = [B.malloc(8 * MiB, AK_KV) for _ in range(2)]
    S = [B.malloc(s, AK_STATIC) for s in (2048, 2048, 2048, 1 << 19, 1024, 4 * MiB + 1024)]
    # 23 allocations so far; the graph adds E, F, 35 temps and 4 permanent buffers = 64.
    B.begin_capture()
    E = B.malloc(H * 2, AK_CAPTURE, "graph")
    B.node("embed", [(E, 0), (S[0], 0), (W[0], 0)], ("toy", "embed"), DLSYM, 1)
    temps = [E]
    n_temp = [18, 17]
    gemm_perm_nodes = {(0, 10), (1, 40)}
    for li in range(2):
        alloc_at = set(rng.choice(np.arange(99), size=n_temp[li], replace=False).tolist())
        for ni in range(99):
            tmpl = _TOY_POOL[int(rng.integers(0, len(_TOY_POOL)))]
            if (li, ni) in gemm_perm_nodes:
                tmpl = "gemm"
            if ni in alloc_at:
                sz = int(rng.choice([H * 2, 3 * H * 2, 2 * I * 2, I * 2, H * 4]))
                temps.append(B.malloc(sz, AK_CAPTURE, "graph"))
            n_words, ppos = TEMPLATES[tmpl]
            pool = temps[-4:] + LW[li] + [KV[li], S[1], S[2], S[3], S[4]]
            ptrs = [(pool[int(rng.integers(0, len(pool)))], 0) for _ in ppos]
            perms = ()
            if (li, ni) in gemm_perm_nodes:
                perms = (B.malloc(4, AK_PERM, "graph"), B.malloc(4, AK_PERM, "graph"))
            fk = ("toy", tmpl, li if tmpl == "gemm" else 0)
            B.node(tmpl, ptrs, fk, TRIGGER if tmpl == "gemm" else DLSYM, 1, perms)
            # free the oldest temp (never E) once more than 4 are alive
            alive = [a for a in temps[1:] if B.a_tf[a] == T_NEVER]
            if len(alive) > 4:
                B.free(alive[0])
    F = B.malloc(H * 2, AK_CAPTURE, "graph")
    B.node("rmsnorm", [(F, 0), (temps[-1], 0), (W[1], 0)], ("toy", "rmsnorm"), DLSYM, 1)
    B.end_capture()
    # the graph's temporaries are released after the capture; its
    # permanent buffers stay
    for a in temps + [F]:
        if B.a_tf[a] == T_NEVER:
            B.free(a)
    B.end_model()
    assert len(B.a_base) == 64, len(B.a_base)


# ---------------------------------------------------------------------------
CONFIGS = {
    "toy": dict(models=None, seed=1),
    "qwen1.5-4b": dict(models=["qwen1.5-4b"], seed=2),
    "llama2-7b": dict(models=["llama2-7b"], seed=3),
    "all10": dict(models=ALL10, seed=4),
    "llama2-13b": dict(models=["llama2-13b"], seed=100),  # C5: seed 100 + gpu index
    # stress: ALL10 with ~8% of all words in-band non-pointer constants (addresses in
    # VA holes and in freed memory, inside [least base, greatest end) of the trace),
    # so the classify prefilter cannot reject them for free
    "all10-inband": dict(models=ALL10, seed=5, rates=(0.08, 0.005, 0.015, 0.0005)),
}


def make_graph_set(config: str, seed: int | None = None, models: list | None = None) -> GraphSet:
    """Build one of the BASELINE.json configurations.

    config: 'toy' | 'qwen1.5-4b' | 'llama2-7b' | 'all10' | 'llama2-13b' | 'all10-inband' (stress) |
    any single model name.
    seed defaults to the config's fixed seed.
    """
    rates = _RATES
    if config in CONFIGS:
        spec = CONFIGS[config]
        mlist = spec["models"] if models is None else models
        seed = spec["seed"] if seed is None else seed
        rates = spec.get("rates", _RATES)
    elif config in MODELS:
        mlist = [config] if models is None else models
        seed = 0 if seed is None else seed
    else:
        raise KeyError(config)
    B = _Builder(seed, rates)
    if mlist is None:
        _run_toy(B)
    else:
        for mi, name in enumerate(mlist):
            _run_model(B, mi, MODELS[name])
    return B.build(config)


def replicate(gs: GraphSet, R: int, va_stride: int = 1 << 44) -> GraphSet:
    """R copies of a graph set as one larger set (SURVEY.md §8(d) sustained mode):
    replica r lives va_stride*r higher in the address space (every address-valued
    word moves with it; plain constants do not), after all events of replica r-1
    in time, with allocation ordinals and kernel-name ids offset by r copies."""
    assert R >= 1
    span = int(max(int(gs.node_t.max(initial=0)), int(gs.allocs["t_alloc"].max(initial=0)),
                   int(gs.capture_t.max(initial=0)),
                   int(np.where(gs.allocs["t_free"] == T_NEVER, 0, gs.allocs["t_free"]).max(initial=0)))) + 1
    assert span * R < T_NEVER
    is_addr = gs.tags != TAG_CONST
    words, tags, tid, toff, offs, nts, fids = [], [], [], [], [np.zeros(1, np.uint64)], [], []
    allocs, new_base, caps = [], [], []
    K = gs.table.size
    for r in range(R):
        d = np.uint64(va_stride * r)
        w = gs.words.copy()
        w[is_addr] += d
        words.append(w)
        tags.append(gs.tags)
        tid.append(np.where(gs.truth_id >= 0, gs.truth_id + r * gs.n_alloc, -1))
        toff.append(gs.truth_off)
        offs.append(gs.node_word_off[1:] + np.uint64(r * gs.n_words))
        nts.append(gs.node_t + np.uint32(r * span))
        fids.append(gs.func_id + np.uint32(r * K))
        a = gs.allocs.copy()
        a["base"] += d
        a["t_alloc"] += np.uint32(r * span)
        never = a["t_free"] == T_NEVER
        a["t_free"] = np.where(never, T_NEVER, a["t_free"] + np.uint32(r * span))
        allocs.append(a)
        new_base.append(gs.new_base + d)
        caps.append(gs.capture_t + np.uint32(r * span))
    return GraphSet(
        name=f"{gs.name}x{R}", words=np.concatenate(words), node_word_off=np.concatenate(offs),
        node_t=np.concatenate(nts), func_id=np.concatenate(fids), allocs=np.concatenate(allocs),
        new_base=np.concatenate(new_base), new_size=np.tile(gs.new_size, R), table=np.tile(gs.table, R),
        func_kind=np.tile(gs.func_kind, R), tags=np.concatenate(tags), truth_id=np.concatenate(tid),
        truth_off=np.concatenate(toff), node_model=np.tile(gs.node_model, R), node_bs=np.tile(gs.node_bs, R),
        node_perm=np.tile(gs.node_perm, R), alloc_kind=np.tile(gs.alloc_kind, R), models=gs.models * R,
        capture_t=np.concatenate(caps))
