// MATERIALIZE: indirect-index-pointer analysis (§4.1) on
// sm_100a.  For every 8-byte word w of node j (launched at t_j), find the
// allocation i live at the launch (t_alloc_i < t_j < t_free_i) whose range
// [base_i, base_i + size_i) holds w ("identical or within the range");
// emit the indirect index pointer table in word order.
//
// Structure of a well-formed trace that the GPU design exploits:
//  * I = allocations live at the LAST launch T_last.  All of them are live at
//    the same instant, so they are pairwise address-disjoint: one list sorted by
//    base answers "which I-allocation holds w" with one search; it is live at
//    t <= T_last iff t_alloc < t.  (Weights, KV cache, static inputs, permanent
//    buffers: ~27k entries for the ten-model set.)
//  * M = every other allocation ("mortal": capture temporaries, warm-up and
//    profiling scratch).  The mortals live at one launch are pairwise disjoint;
//    a chunk's window (~60 entries for the ten-model set) holds exactly the
//    mortals live at one of its launches, found by a descent of the MORTAL TREE
//    (a 32-ary max tree over ordinals: leaf = t_free of a mortal, node = max
//    over its ordinals + the first ordinal's t_alloc); a word is looked up among
//    the entries live at its node (about four) by a range test.
//  * Well-formedness (no two simultaneously-live allocations overlap) is checked
//    exactly: I-I by adjacency of the sorted list, M-I with per-32-entry
//    min(t_alloc) / max(t_free) summaries over the address run a mortal meets,
//    M-M per block of 32 ordinals against the mortals the tree reports live when
//    they are allocated.
// Pipeline (the synchronous entry adds one host read at the end):
//   memset -> k_trace -> k_classify -> (after k_rank) k_iresolve -> k_emit ....(join) [-> k_result]
//   side (high priority):  k_isort -> k_rank --^
//   low (default priority): k_check_mm ... (after k_rank) k_check_mi ------------------^
//   k_trace      [nodes] CSR / launch-order checks, first/last node of each chunk and
//                their launch positions; [allocs] trace checks, I/M split, the
//                mortal tree, prefilter bounds, I compaction (ordinal order)
//   k_isort      I keys sorted in tiles of 1024 (register bitonic per warp + merges)
//   k_rank       global rank of every I key -> the sorted I arrays, fences, summaries
//   k_classify   one CTA per 2048-word chunk: TMA copy of the words (before the
//                wait), node starts, the window by a tree query, candidate
//                compaction, live masks, lookups; per warp: records and I-list
//                queue entries into its regions, mask words, slot count
//   k_check_mm   M-M overlap check (tree descent per warp)
//   k_check_mi   M-I and I-I overlap checks
//   k_iresolve   queued candidates against the sorted I list
//   k_emit       chunk_base (two-level prefix) and the records compacted into the
//                slot table
#include <algorithm>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace medusa {
namespace {

MEDUSA_TL_DEFINE

constexpr uint32_t ST_INVALID = 1, ST_TRACE = 2, ST_OVERFLOW = 4;
constexpr int kThreads = 256;
constexpr int kAblk = 32;          // allocation ordinals per overlap-check block (one warp)
constexpr int kChkCap = 64;        // registered mortals staged per warp batch
constexpr int kFenceCap = 2048;    // I-list fences (every stride-th sorted base): k_iresolve holds them in
                                   //  shared memory (8192 searched through L1, and 4096 in shared memory
                                   //  with a CTA's two chunks overlapped, measured slower: DESIGN.md §6)
constexpr int kWinCap = 96;        // mortal-window entries per batch (<= 4 per lane of one warp; 96 keeps 7 classify CTAs per SM)
constexpr int kWordsPerThread = MEDUSA_CHUNK_WORDS / kThreads;  // 8
constexpr int kWarps = kThreads / 32;
constexpr int kIBlk = 32;          // I-list summary block
constexpr int kNodeGrp = 128;      // nodes per live-mask group (a chunk holds ~90 nodes in the BASELINE sets)

struct Ctl {
    unsigned int status;
    unsigned int nI;
    unsigned int pad0;
    unsigned int pad1;
    unsigned long long gmin_c;  // ~(least base) via atomicMax
    unsigned long long gmax;    // greatest end
    unsigned long long n_slots;
    unsigned int need_pw, pad2;           // entries per warp region a call needed (set only on overflow)
};

struct IRest {  // I-list entry (sorted order), base kept in a separate array
    uint64_t end;
    uint32_t t_alloc;
    uint32_t id;
};

struct IQ {  // a candidate word for the I-list search (k_iresolve)
    uint64_t x;  // the word
    uint32_t g;  // its index in the image
    uint32_t t;  // launch position of its node
};

// The mortal tree: a 32-ary max tree over allocation ordinals.
// Leaf i = {v_i, t_alloc_i} with v_i = t_free_i for a mortal (non-empty, not in
// I) and 0 otherwise; node k of level l >= 1 covers ordinals [k 32^l, (k+1) 32^l)
// and holds {max v, t_alloc of its first ordinal}.  "The mortals allocated before
// T1 and freed after T0" is a descent that keeps the nodes with max v > T0 and
// first t_alloc < T1 (t_alloc increases with the ordinal on a well-formed trace).
constexpr int kMaxLevels = 6;  // 32^5 > 2^24 allocations
struct Tree {
    uint2* leaf;                  // [n] {v, t_alloc}
    ulonglong2* leaf_be;          // [n] {base, base + size}: a kept leaf is a window entry as loaded
    uint2* node;                  // levels 1..top, level l at node + off[l]
    uint32_t off[kMaxLevels + 1]; // off[1] = 0
    uint32_t cnt[kMaxLevels + 1]; // nodes of level l (cnt[0] = n)
    uint32_t top;                 // the level with <= 32 nodes (0 if n <= 32)
    int32_t l0;                   // a query's start level: the highest with <= kThreads nodes (set on the host)
};

struct Dev {  // scratch of one call (device pointers)
    Ctl* ctl;
    uint2 *jf, *jl;                              // [C] first / last node of each chunk and its launch position
    Tree tree;
    unsigned long long* chunk_sup;               // [C/256+1] slots per 256 chunks
    uint32_t *blk_min_ta_c, *blk_max_tf;         // [n/32+1] (zeroed; min kept as ~max(~t))
    uint64_t *sk0, *sk;                          // [n] I keys (base): compacted by k_trace / sorted tiles
    uint32_t *sv0, *sv;                          // [n] their allocation ordinals
    uint32_t* icnt;                              // [n/256+1] I keys of each k_trace alloc CTA (ordered mode)
    uint64_t* tmax_k;                            // [n/1024+1] greatest key of each sorted tile
    uint32_t* tmax_v;
    uint64_t* samp_k;                            // [n/64+1] every 64th key of each sorted tile
    uint32_t* samp_v;
    uint64_t* i_base;                            // [n]
    IRest* i_rest;                               // [n]
    uint32_t* i_tf;                              // [n]
    uint64_t* fence;                             // [kFenceCap]
    uint32_t* chunk_cnt;                         // [C] slots per chunk
    // Warp-local record regions: classify warp w of chunk c (its
    // 256 words) owns entries [(8c + w) cap_pw, (8c + w + 1) cap_pw) of each,
    // filled in word order
    uint64_t* rec;                               // records of the window hits
    IQ* queue;                                   // candidates left for the I-list search; k_iresolve
                                                 //  overwrites a hit's word (x) with its record
    uint32_t cap_pw;                             // entries per warp region (128; 256 after an overflow)
    uint32_t* qcnt;                              // [C * 8] queue entries of classify warp w of chunk c
    uint32_t *imask, *qmask;                     // [ceil(n_words/32)] words resolved by the I list / queued
};

struct P {  // kernel parameters
    MaterializeArgs a;
    Dev d;
    uint32_t C, nb;              // chunks, check blocks (32 ordinals each)
    uint32_t node_ctas;          // k_trace: CTAs with the node role
    uint32_t alloc_ctas;         // k_trace: CTAs with the allocation role
    uint32_t ordered;            // I keys compacted in ordinal order (k_isort gathers them by the
                                 //  CTA prefix of icnt); else in atomic order (very large traces)
};

__device__ __forceinline__ void flag(Ctl* c, unsigned int bit) { atomicOr(&c->status, bit); }

__device__ __forceinline__ bool kv_less(uint64_t ka, uint32_t va, uint64_t kb, uint32_t vb) {
    return ka < kb || (ka == kb && va < vb);
}

__device__ __forceinline__ uint64_t warp_min_u64(uint64_t v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v = min(v, (uint64_t)__shfl_xor_sync(0xffffffffu, v, d));
    return v;
}
__device__ __forceinline__ uint64_t warp_max_u64(uint64_t v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v = max(v, (uint64_t)__shfl_xor_sync(0xffffffffu, v, d));
    return v;
}

// every stride-th sorted I base is a fence; the stride is a multiple of 4 so a
// group [j stride, (j + 1) stride) of the sorted bases is whole 32-byte blocks
// (the i_base array is 256-byte aligned and padded)
__device__ __forceinline__ uint32_t fence_stride(uint32_t nI) {
    return 4u * max(1u, (nI + 4u * kFenceCap - 1) / (4u * kFenceCap));  // (>= 4 also for an empty list)
}

// Sum of cnt[0, k) of a two-level counter (sup[g] = sum of cnt[256g, 256g + 256)):
// at most k/256 + 255 loads, spread over the CTA, and one reduction; every thread
// receives the value.  Call with the whole CTA (blockDim.x == kThreads == 256).
static_assert(kThreads == 256, "block_prefix covers one 256-key group per pass");
__device__ __forceinline__ unsigned long long block_prefix(const uint32_t* cnt, const unsigned long long* sup,
                                                           uint32_t k) {
    __shared__ unsigned long long s_r[kWarps];
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t g = k >> 8;
    unsigned long long acc = 0;
    for (uint32_t q = threadIdx.x; q < g; q += kThreads) acc += __ldcg(sup + q);
    const uint32_t j = (g << 8) + threadIdx.x;
    if (j < k) acc += __ldcg(cnt + j);
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, d);
    if (lane == 0) s_r[warp] = acc;
    __syncthreads();
    unsigned long long t = 0;
#pragma unroll
    for (int w = 0; w < kWarps; ++w) t += s_r[w];
    return t;  // (called once per CTA: s_r is not rewritten, no barrier after the reads)
}

// one allocation record through the read-only path
__device__ __forceinline__ medusa_alloc ld_alloc(const medusa_alloc* q) {
    const unsigned long long* w = reinterpret_cast<const unsigned long long*>(q);
    const unsigned long long b = __ldg(w), z = __ldg(w + 1), t = __ldg(w + 2);
    medusa_alloc x;
    x.base = b;
    x.size = z;
    x.t_alloc = (uint32_t)t;
    x.t_free = (uint32_t)(t >> 32);
    return x;
}


// ----------------------------------------------------------------------------
// 0. k_zero: the call's zeroed scratch (counters, check summaries, tree nodes) as
//    the first kernel, so that k_trace is its programmatic successor: k_trace's
//    CTAs load their records while it runs (a memset node measured ~2 us more
//    in front of the first CTA)
__global__ void __launch_bounds__(kThreads) k_zero(uint4* z, size_t n16) {
    // launched programmatically: the previous kernels (the last of an earlier call
    // may still read this scratch; one may have written the image) complete first,
    // then k_trace and k_classify may start and read the inputs
    pdl_wait();
    pdl_trigger();
    for (size_t k = (size_t)blockIdx.x * kThreads + threadIdx.x; k < n16; k += (size_t)gridDim.x * kThreads)
        z[k] = make_uint4(0u, 0u, 0u, 0u);
}

// ----------------------------------------------------------------------------
// 1. k_trace
// node i of the CSR (o0 = node_off[i], o1 = node_off[i + 1], t0 / t1 = the launch
// positions of nodes i and i + 1): the CSR / launch-order checks and the chunks
// whose first or last word it holds
__device__ __forceinline__ void nodes_role(const P& p, uint64_t i, uint64_t o0, uint64_t o1, uint32_t t0, uint32_t t1) {
    const MaterializeArgs& a = p.a;
    const uint32_t N = a.n_nodes;
    if (i > N) return;
    if (i == 0 && o0 != 0) flag(p.d.ctl, ST_INVALID);
    if (i == N) {
        if (o0 != a.n_words) flag(p.d.ctl, ST_INVALID);
        return;
    }
    if (o1 < o0) { flag(p.d.ctl, ST_INVALID); return; }
    if (i + 1 < N && !(t0 < t1)) flag(p.d.ctl, ST_INVALID);
    if (o1 == o0 || o1 > a.n_words) return;
    // node i writes the chunks whose first or last word it holds
    for (uint64_t c = o0 / kChunkWords; c <= (o1 - 1) / kChunkWords; ++c) {
        const uint64_t cs = c * kChunkWords;
        const uint64_t ce = min(cs + kChunkWords, a.n_words) - 1;
        if (o0 <= cs) p.d.jf[c] = make_uint2((uint32_t)i, t0);
        if (ce < o1) p.d.jl[c] = make_uint2((uint32_t)i, t0);
    }
}

constexpr int kNodesPerThread = 4;  // node role of k_trace (keeps its grid inside one wave)

// One allocation per thread: the trace checks (R-Q7, R-Q9), the I / M split, the
// mortal tree (leaf, level 1 by the warp, higher levels by one atomic per CTA),
// the prefilter bounds and the I compaction.  One coalesced record load, no search.
__device__ void allocs_role(const P& p, uint32_t cta) {
    const MaterializeArgs& a = p.a;
    const Tree& T = p.d.tree;
    const uint32_t i0 = cta * blockDim.x;
    const uint32_t i = i0 + threadIdx.x;
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t N = a.n_nodes;
    const bool valid = i < a.n_alloc;
    unsigned long long tl_p = TL_NOW();
    medusa_alloc x{};
    if (valid) x = ld_alloc(a.alloc + i);
    const uint32_t t_last = N ? __ldg(a.node_t + N - 1) : 0;
    uint32_t ta_next = __shfl_down_sync(0xffffffffu, x.t_alloc, 1);  // the next ordinal's t_alloc
    if (lane == 31 && i + 1 < a.n_alloc) ta_next = (uint32_t)__ldg(reinterpret_cast<const unsigned long long*>(a.alloc + i + 1) + 2);
    pdl_wait();  // (k_zero: the counters and tree nodes below are zero)
    bool isI = false;
    uint32_t v = 0;  // leaf value: t_free of a mortal, else 0
    if (valid) {
        if (x.size > (1ull << MEDUSA_OFF_BITS) || x.base + x.size < x.base) flag(p.d.ctl, ST_INVALID);
        if (!(x.t_alloc < x.t_free)) flag(p.d.ctl, ST_TRACE);
        if (i + 1 < a.n_alloc && !(x.t_alloc < ta_next)) flag(p.d.ctl, ST_TRACE);
        if (x.size != 0) {
            isI = N && x.t_alloc < t_last && t_last < x.t_free;
            if (!isI) v = x.t_free;
        }
        T.leaf[i] = make_uint2(v, x.t_alloc);
        T.leaf_be[i] = make_ulonglong2(x.base, x.base + x.size);
    }
    TL_PHASE(1, 20, tl_p);  // record load, checks
    // the mortal tree above the leaves: level 1 = this warp's 32 ordinals
    const uint32_t wmax = __reduce_max_sync(0xffffffffu, v);
    if (T.top >= 1 && lane == 0 && valid) T.node[T.off[1] + (i >> 5)] = make_uint2(wmax, x.t_alloc);
    // levels >= 2: the first ordinal's t_alloc directly, the max by one atomic per CTA
    // (a CTA's 256 ordinals lie inside one node of every level >= 2)
    for (uint32_t l = 2; l <= T.top; ++l)
        if (valid && (i & ((1u << (5 * l)) - 1)) == 0) T.node[T.off[l] + (i >> (5 * l))].y = x.t_alloc;
    // CTA-aggregated (one global atomic per CTA, not per warp: these are the same
    // addresses for every CTA): I positions, global prefilter bounds, upper tree levels
    __shared__ uint32_t s_ni, s_base, s_wmax[kWarps], s_wi[kWarps];
    __shared__ unsigned long long s_mn, s_mx;
    const uint32_t bal = __ballot_sync(0xffffffffu, isI);
    if (threadIdx.x == 0) { s_mn = ~0ull; s_mx = 0; }
    if (lane == 0) { s_wmax[warp] = wmax; s_wi[warp] = __popc(bal); }
    __syncthreads();
    uint32_t wpos = 0;  // the warp's first I key in the CTA: ordinal order
#pragma unroll
    for (int w = 0; w < kWarps; ++w) wpos += (uint32_t)w < warp ? s_wi[w] : 0u;
    const bool live = valid && x.size != 0;
    const uint64_t mn = warp_min_u64(live ? x.base : ~0ull);
    const uint64_t mx = warp_max_u64(live ? x.base + x.size : 0ull);
    if (lane == 0 && mx) {
        atomicMin(&s_mn, (unsigned long long)mn);
        atomicMax(&s_mx, (unsigned long long)mx);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t ni = 0;
#pragma unroll
        for (int w = 0; w < kWarps; ++w) ni += s_wi[w];
        s_ni = ni;
        // ordered: the CTA's keys at its own region, k_isort finds them by the CTA
        // prefix of icnt; else one atomic hands out positions
        if (p.ordered) { s_base = cta * kThreads; p.d.icnt[cta] = ni; }
        if (ni) {  // (ordered: a reduction, nothing to wait for; else the CTA's positions)
            if (p.ordered) atomicAdd(&p.d.ctl->nI, ni);
            else s_base = atomicAdd(&p.d.ctl->nI, ni);
        }
        if (s_mx) {
            atomicMax(&p.d.ctl->gmin_c, ~s_mn);
            atomicMax(&p.d.ctl->gmax, s_mx);
        }
        uint32_t cmax = 0;
#pragma unroll
        for (int w = 0; w < kWarps; ++w) cmax = max(cmax, s_wmax[w]);
        if (cmax)
            for (uint32_t l = 2; l <= T.top; ++l) atomicMax(&T.node[T.off[l] + (i0 >> (5 * l))].x, cmax);
    }
    __syncthreads();
    if (isI) {
        const uint32_t pos = s_base + wpos + __popc(bal & lanemask_lt());
        p.d.sk0[pos] = x.base;
        p.d.sv0[pos] = i;
    }
    TL_PHASE(1, 22, tl_p);  // tree, prefilter bounds, I compaction
}

__global__ void __launch_bounds__(kThreads, 8) k_trace(P p) {
    const unsigned long long tl0 = TL_NOW();
    // k_classify's CTAs may start in the slots this grid leaves free and issue
    // their word copies; they read nothing of this grid before griddepcontrol.wait
    pdl_trigger();
    if (blockIdx.x < p.node_ctas) {  // kNodesPerThread nodes per thread, CTA-strided
        // every node's offsets and launch positions loaded in one round, then the checks
        const uint32_t N = p.a.n_nodes;
        uint64_t o0[kNodesPerThread], o1[kNodesPerThread];
        uint32_t t0[kNodesPerThread], t1[kNodesPerThread];
#pragma unroll
        for (int k = 0; k < kNodesPerThread; ++k) {
            const uint64_t i = ((uint64_t)blockIdx.x * kNodesPerThread + k) * blockDim.x + threadIdx.x;
            o0[k] = i <= N ? __ldg(p.a.node_off + i) : 0ull;
            o1[k] = i < N ? __ldg(p.a.node_off + i + 1) : 0ull;
            t0[k] = i < N ? __ldg(p.a.node_t + i) : 0u;
            t1[k] = i + 1 < N ? __ldg(p.a.node_t + i + 1) : 0u;
        }
        pdl_wait();  // (k_zero)
#pragma unroll
        for (int k = 0; k < kNodesPerThread; ++k)
            nodes_role(p, ((uint64_t)blockIdx.x * kNodesPerThread + k) * blockDim.x + threadIdx.x, o0[k], o1[k], t0[k],
                       t1[k]);
        TL_REC(1, 0, tl0);
    } else {
        allocs_role(p, blockIdx.x - p.node_ctas);
        TL_REC(1, 1, tl0);
    }
}

// ----------------------------------------------------------------------------
// 2. k_isort: sort tiles of I keys by (base, index)

// the I entry of sorted position r: arrays, fence, block summaries
__device__ __forceinline__ void write_i_entry(const P& p, uint32_t r, uint32_t nI, uint32_t id, const medusa_alloc& x) {
    MCHECK(r < nI && id < p.a.n_alloc);
    p.d.i_base[r] = x.base;
    p.d.i_rest[r] = IRest{x.base + x.size, x.t_alloc, id};
    p.d.i_tf[r] = x.t_free;
    const uint32_t stride = fence_stride(nI);
    if (r % stride == 0) p.d.fence[r / stride] = x.base;
    atomicMax(&p.d.blk_min_ta_c[r / kIBlk], ~x.t_alloc);
    atomicMax(&p.d.blk_max_tf[r / kIBlk], x.t_free);
}

// write_i_entry by the active lanes of a warp, the block summaries combined per
// block first (k_rank: a warp's 32 keys mostly take consecutive ranks, so one
// pair of atomics per block instead of one per key -- the per-key atomics on the
// same block cost k_rank ~1.3 us of its span beside k_classify, measured)
// (act: the calling lanes, all of which make this call)
__device__ __forceinline__ void write_i_entry_warp(const P& p, uint32_t r, uint32_t nI, uint32_t id, const medusa_alloc& x,
                                                   uint32_t act) {
    MCHECK(r < nI && id < p.a.n_alloc && ((act >> (threadIdx.x & 31)) & 1u));
    p.d.i_base[r] = x.base;
    p.d.i_rest[r] = IRest{x.base + x.size, x.t_alloc, id};
    p.d.i_tf[r] = x.t_free;
    const uint32_t stride = fence_stride(nI);
    if (r % stride == 0) p.d.fence[r / stride] = x.base;
    const uint32_t b = r / kIBlk;
    const uint32_t grp = __match_any_sync(act, b);
    const uint32_t mn_c = __reduce_max_sync(grp, ~x.t_alloc);  // (min t_alloc kept as the max of its complement)
    const uint32_t mx = __reduce_max_sync(grp, x.t_free);
    if ((grp & lanemask_lt()) == 0) {
        atomicMax(&p.d.blk_min_ta_c[b], mn_c);
        atomicMax(&p.d.blk_max_tf[b], mx);
    }
}

// Bitonic sort of 32*E (key, val) pairs held E per lane (element lane*E + r),
// ascending by (key, val); shuffles and register compare-exchanges only.
template <int E>
__device__ __forceinline__ void warp_bitonic_kv(uint64_t (&k)[E], uint32_t (&v)[E]) {
    const uint32_t lane = threadIdx.x & 31;
#pragma unroll
    for (uint32_t size = 2; size <= 32u * E; size <<= 1) {
#pragma unroll
        for (uint32_t j = size >> 1; j > 0; j >>= 1) {
            if (j >= (uint32_t)E) {
                const uint32_t lj = j / E;
                const bool lower = (lane & lj) == 0;
#pragma unroll
                for (int r = 0; r < E; ++r) {
                    const uint32_t e = lane * E + r;
                    const uint64_t ok = __shfl_xor_sync(0xffffffffu, k[r], lj);
                    const uint32_t ov = __shfl_xor_sync(0xffffffffu, v[r], lj);
                    const bool up = (e & size) == 0;
                    const bool other_less = kv_less(ok, ov, k[r], v[r]);
                    if ((lower == up) ? other_less : !other_less) { k[r] = ok; v[r] = ov; }
                }
            } else {
#pragma unroll
                for (int r = 0; r < E; ++r) {
                    const int r2 = r ^ (int)j;
                    if (r2 > r && kv_less(k[r2], v[r2], k[r], v[r]) == (((lane * E + r) & size) == 0)) {
                        const uint64_t tk = k[r]; k[r] = k[r2]; k[r2] = tk;
                        const uint32_t tv = v[r]; v[r] = v[r2]; v[r2] = tv;
                    }
                }
            }
        }
    }
}

// ----------------------------------------------------------------------------
// 2a. k_isort (side stream, after k_trace): tile t = the I keys at compacted
//     positions [t S, t S + S), S = kIsortTile = 1024 (k_trace compacts the I
//     allocations: non-empty, t_alloc < T_last < t_free).  Sorted by (base,
//     ordinal): a register bitonic sort of 128 keys per warp, then three
//     merge-path rounds through shared memory (128 -> 256 -> 512 -> 1024), four
//     keys per thread held in registers between rounds.  A single tile is the
//     whole list: its I entries are written here and k_rank has nothing to do.  Otherwise the sorted tile goes
//     to sk / sv and every kSampleStride-th key is its sample for k_rank.
constexpr int kIsortThreads = 256;  // (1024-thread CTAs measured slower: they find no slot beside
                                     //  the classify CTAs, and one CTA sorting 3-4k keys is a long chain)
#ifndef MEDUSA_ISORT_PER
#define MEDUSA_ISORT_PER 4
#endif
constexpr int kSortPer = MEDUSA_ISORT_PER;                   // keys per thread in registers
constexpr int kIsortTile = kIsortThreads * kSortPer;         // 1024
constexpr int kSampleStride = kIsortTile / 64 > 32 ? kIsortTile / 64 : 32;  // <= 64 samples per tile
struct ISortShared {
    uint64_t k[kIsortTile];
    uint32_t v[kIsortTile];
};
constexpr size_t kIsortSmem = sizeof(ISortShared);

constexpr uint32_t kOrderedCtas = 16384;  // ordered compaction up to 16384 k_trace alloc CTAs (4 M allocations)

__global__ void __launch_bounds__(kIsortThreads) k_isort(P p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    ISortShared& S = *reinterpret_cast<ISortShared*>(smem_raw);
    uint32_t* s_pre = reinterpret_cast<uint32_t*>(smem_raw + sizeof(ISortShared));  // [alloc_ctas + 1]
    __shared__ uint32_t s_wsum[kIsortThreads / 32];
    const unsigned long long tl0 = TL_NOW();
    unsigned long long tl_p = tl0;
    const uint32_t n = p.d.ctl->nI;
    const uint32_t t0 = blockIdx.x * kIsortTile;
    if (t0 >= n) return;
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (p.ordered) {  // where each k_trace CTA's I keys start in ordinal order (exclusive prefix of icnt)
        const uint32_t nbk = p.alloc_ctas;
        const uint32_t per = (nbk + kIsortThreads - 1) / kIsortThreads;
        const uint32_t b0 = min(tid * per, nbk), b1 = min(b0 + per, nbk);
        uint32_t sum = 0;
        for (uint32_t b = b0; b < b1; ++b) { const uint32_t c = __ldcg(p.d.icnt + b); s_pre[b] = sum; sum += c; }
        uint32_t incl = sum;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= (uint32_t)d) incl += y;
        }
        if (lane == 31) s_wsum[warp] = incl;
        __syncthreads();
        uint32_t before = incl - sum;
        for (uint32_t w = 0; w < warp; ++w) before += s_wsum[w];
        for (uint32_t b = b0; b < b1; ++b) s_pre[b] += before;
        if (tid == kIsortThreads - 1) s_pre[nbk] = before + sum;
        __syncthreads();
    }
    const uint32_t o = tid * kSortPer;  // this thread's consecutive elements
    uint64_t k[kSortPer];
    uint32_t v[kSortPer];
    // (ordered) the k_trace CTA holding compacted position g = last b with s_pre[b]
    // <= g: one binary search for the thread's first position, then a forward step
    // per following one (its kSortPer positions are consecutive)
    uint32_t lo = 0;
    if (p.ordered && t0 + o < n) {
        uint32_t hi = p.alloc_ctas;
        const uint32_t g = t0 + o;
        while (hi - lo > 1) { const uint32_t mid = (lo + hi) >> 1; if (s_pre[mid] <= g) lo = mid; else hi = mid; }
    }
#pragma unroll
    for (int r = 0; r < kSortPer; ++r) {
        const uint32_t g = t0 + o + r;
        uint32_t q = g;
        if (p.ordered && g < n) {
            while (lo + 1 < p.alloc_ctas && s_pre[lo + 1] <= g) ++lo;  // (empty CTAs share a prefix value)
            q = lo * kThreads + (g - s_pre[lo]);
            MCHECK(lo < p.alloc_ctas && g >= s_pre[lo] && g - s_pre[lo] < (uint32_t)kThreads && q < p.a.n_alloc);
        }
        k[r] = g < n ? __ldcg(p.d.sk0 + q) : ~0ull;
        v[r] = g < n ? __ldcg(p.d.sv0 + q) : 0xFFFFFFFFu;
    }
    warp_bitonic_kv<kSortPer>(k, v);
    TL_PHASE(2, 30, tl_p);  // load + warp bitonic
#pragma unroll 1
    for (uint32_t run = 32 * kSortPer; run < kIsortTile; run <<= 1) {
#pragma unroll
        for (int r = 0; r < kSortPer; ++r) { S.k[o + r] = k[r]; S.v[o + r] = v[r]; }
        __syncthreads();
        const uint32_t a0 = o / (2 * run) * (2 * run), b0 = a0 + run;
        const uint32_t d = o - a0;
        uint32_t lo = d > run ? d - run : 0, hi = min(d, run);
        while (lo < hi) {  // merge path: A elements among the first d of the merged pair
            const uint32_t mid = (lo + hi) >> 1;
            const uint32_t pb = b0 + d - 1 - mid, pa = a0 + mid;
            const uint64_t x = S.k[pa], y = S.k[pb];  // values only break key ties
            if (x < y || (x == y && S.v[pa] < S.v[pb])) lo = mid + 1; else hi = mid;
        }
        uint32_t ia = lo, ib = d - lo;
#pragma unroll
        for (int r = 0; r < kSortPer; ++r) {
            const uint32_t pa = a0 + min(ia, run - 1), pb = b0 + min(ib, run - 1);
            const uint64_t ka = S.k[pa], kb = S.k[pb];
            const uint32_t va = S.v[pa], vb = S.v[pb];
            const bool takeA = ib >= run || (ia < run && kv_less(ka, va, kb, vb));
            k[r] = takeA ? ka : kb;
            v[r] = takeA ? va : vb;
            if (takeA) ++ia; else ++ib;
        }
        __syncthreads();
    }
    TL_PHASE(2, 31, tl_p);  // shared-memory merges
    const bool single = n <= (uint32_t)kIsortTile;  // one tile: its order is final
    medusa_alloc x[kSortPer];
    if (single) {  // all record loads first (independent), then the writes
#pragma unroll
        for (int r = 0; r < kSortPer; ++r)
            if (o + r < n) x[r] = ld_alloc(p.a.alloc + v[r]);
    }
#pragma unroll
    for (int r = 0; r < kSortPer; ++r) {
        const uint32_t q = o + r;
        if (t0 + q >= n) break;
        if (single) {
            write_i_entry(p, q, n, v[r], x[r]);
        } else {
            p.d.sk[t0 + q] = k[r];
            p.d.sv[t0 + q] = v[r];
            if ((q % kSampleStride) == 0) {  // the tile's sample for k_rank
                p.d.samp_k[t0 / kSampleStride + q / kSampleStride] = k[r];
                p.d.samp_v[t0 / kSampleStride + q / kSampleStride] = v[r];
            }
            if (t0 + q + 1 == min(t0 + kIsortTile, n)) {  // the tile's greatest key
                p.d.tmax_k[blockIdx.x] = k[r];
                p.d.tmax_v[blockIdx.x] = v[r];
            }
        }
    }
    TL_REC(2, 0, tl0);
    pdl_trigger();
}

// ----------------------------------------------------------------------------
// 2b. k_rank (after k_isort, only with more than one tile): global rank of every
//     I key = its index in its sorted tile + the count of smaller keys in every
//     other tile.  One CTA per range of 32 consecutive keys of one tile (one key
//     per lane); warp w counts against tiles b = w, w + 8, ... (their key ranges
//     come in with one load round, lane t holding tile w + 8t): the tile's <= 32
//     samples (every 32nd key) come in with one coalesced load and locate, by a
//     shuffle search, the 32-key block of the tile holding each lane's lower
//     bound; the block comes in with one more coalesced load and a shuffle
//     search finishes the count.  A tile whose key range lies wholly above or
//     below the 32 keys is counted from its least and greatest key alone (the I
//     keys are compacted in ordinal order, so with several models in one set most
//     tiles hold another model's disjoint address region).  The counts of the 8
//     warps meet in shared memory; warp 0 writes the 32 I entries (with ordered
//     keys, their block summaries combined per block: write_i_entry_warp).
__device__ __forceinline__ bool kv_lt_lane(uint64_t k, uint32_t v, uint32_t src, uint64_t xk, uint32_t xv) {
    const uint64_t sk = __shfl_sync(0xffffffffu, k, src);
    const uint32_t sv = __shfl_sync(0xffffffffu, v, src);
    return kv_less(sk, sv, xk, xv);
}

// number of the <= 64 ascending entries (entry e: lane e % 32 of half e / 32) that
// are below (xk, xv) -- this lane's key; ne = entries present
__device__ __forceinline__ uint32_t count_lt64(uint64_t k0, uint32_t v0, uint64_t k1, uint32_t v1, uint32_t ne,
                                               uint64_t xk, uint32_t xv) {
    const bool hi_half = ne > 32 && kv_lt_lane(k1, v1, 0, xk, xv);  // entry 32 < x
    // count below x inside the lane's half (32 ascending entries); the source
    // lane's value of BOTH halves is fetched, the lane picks
    uint32_t lo = 0, hi = 32;
#pragma unroll
    for (int st = 0; st < 6; ++st) {
        const uint32_t mid = (lo + hi) >> 1;
        const bool lt0 = kv_lt_lane(k0, v0, min(mid, 31u), xk, xv);
        const bool lt1 = kv_lt_lane(k1, v1, min(mid, 31u), xk, xv);
        const bool lt = hi_half ? lt1 : lt0;
        if (lo < hi) { if (lt) lo = mid + 1; else hi = mid; }
    }
    const uint32_t c = (hi_half ? 32 : 0) + lo;
    return c > ne ? ne : c;
}

__global__ void __launch_bounds__(kThreads, 8) k_rank(P p) {
    __shared__ uint32_t s_cnt[kWarps][32];
    const unsigned long long tl0 = TL_NOW();
    pdl_wait();
    const uint32_t nI = p.d.ctl->nI;
    const uint32_t T = (nI + kIsortTile - 1) / kIsortTile;
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // ranges of 32 keys, grid-stride (the grid is sized by the allocation count)
    for (uint32_t g0 = blockIdx.x * 32; T > 1 && g0 < nI; g0 += gridDim.x * 32) {
        const uint32_t ta = g0 / kIsortTile;
        const uint32_t g = g0 + lane;
        const bool has = g < nI;
        const uint64_t xk = has ? __ldcg(p.d.sk + g) : ~0ull;
        const uint32_t xv = has ? __ldcg(p.d.sv + g) : 0xFFFFFFFFu;
        uint32_t cnt = 0;
        // the key ranges of this warp's tiles (warp, warp + 8, ...), lane t holding the
        // t-th: one load round for all of them (up to 32 per pass)
        uint64_t bmnk = 0, bmxk = 0;
        uint32_t bmnv = 0, bmxv = 0;
        uint32_t tpass = 0;  // the pass of 32 tiles whose bounds the lanes hold
        auto load_bounds = [&](uint32_t pass) {
            const uint32_t tl = warp + (pass * 32 + lane) * kWarps;
            if (tl < T) {
                const uint32_t sl = tl * kIsortTile / kSampleStride;
                bmnk = __ldcg(p.d.samp_k + sl); bmnv = __ldcg(p.d.samp_v + sl);
                bmxk = __ldcg(p.d.tmax_k + tl); bmxv = __ldcg(p.d.tmax_v + tl);
            }
        };
        load_bounds(0);
        for (uint32_t tb = warp, ti = 0; tb < T; tb += kWarps, ++ti) {
            if (ti / 32 != tpass) load_bounds(tpass = ti / 32);  // (more than 256 tiles)
            const uint64_t mnk = __shfl_sync(0xffffffffu, bmnk, ti % 32), mxk = __shfl_sync(0xffffffffu, bmxk, ti % 32);
            const uint32_t mnv = __shfl_sync(0xffffffffu, bmnv, ti % 32), mxv = __shfl_sync(0xffffffffu, bmxv, ti % 32);
            if (tb == ta) continue;
            const uint32_t b0 = tb * kIsortTile, nb = min((uint32_t)kIsortTile, nI - b0);
            const uint32_t ns = (nb + kSampleStride - 1) / kSampleStride;  // samples of tile tb (<= 64)
            const uint32_t s0 = b0 / kSampleStride;
            {  // the tile's key range: lanes below its least key count 0, above its greatest nb
                const bool above = has && kv_less(mxk, mxv, xk, xv);
                const bool below = !has || kv_less(xk, xv, mnk, mnv);
                if (__all_sync(0xffffffffu, above || below)) {  // (ordered I keys: most tiles of the ten-model set)
                    cnt += above ? nb : 0u;
                    continue;
                }
            }
            uint64_t sk0 = ~0ull, sk1 = ~0ull;
            uint32_t sv0 = 0xFFFFFFFFu, sv1 = 0xFFFFFFFFu;
            if (lane < ns) { sk0 = __ldcg(p.d.samp_k + s0 + lane); sv0 = __ldcg(p.d.samp_v + s0 + lane); }
            if (lane + 32 < ns) { sk1 = __ldcg(p.d.samp_k + s0 + lane + 32); sv1 = __ldcg(p.d.samp_v + s0 + lane + 32); }
            // j = #samples < x: the lower bound of x lies in block j - 1 (j >= 1)
            const uint32_t j = count_lt64(sk0, sv0, sk1, sv1, ns, xk, xv);
            // lane l's lower bound lies in block j_l - 1 (ascending over the lanes).
            // Few distinct blocks (the usual case): load each with one coalesced
            // load and count by a shuffle search; otherwise every lane searches its
            // own block in memory (6 dependent loads).
            const uint32_t blk = j ? j - 1 : 0xFFFFFFFFu;
            const bool act = has && j;
            const uint32_t prev = __shfl_up_sync(0xffffffffu, blk, 1);
            const uint32_t n_runs = __popc(__ballot_sync(0xffffffffu, act && (lane == 0 || prev != blk)));
            uint32_t c = 0;
            if (n_runs <= 2) {
                uint32_t pending = __ballot_sync(0xffffffffu, act);
                while (pending) {
                    const uint32_t bl = __shfl_sync(0xffffffffu, blk, __ffs(pending) - 1);
                    const uint32_t q0 = bl * kSampleStride, ne = min((uint32_t)kSampleStride, nb - q0);
                    const uint32_t qa = q0 + lane, qb = q0 + 32 + lane;
                    const uint64_t ka = qa < nb ? __ldcg(p.d.sk + b0 + qa) : ~0ull;
                    const uint32_t va = qa < nb ? __ldcg(p.d.sv + b0 + qa) : 0xFFFFFFFFu;
                    const bool two = kSampleStride > 32 && qb < nb;
                    const uint64_t kb = two ? __ldcg(p.d.sk + b0 + qb) : ~0ull;
                    const uint32_t vb = two ? __ldcg(p.d.sv + b0 + qb) : 0xFFFFFFFFu;
                    const uint32_t below = count_lt64(ka, va, kb, vb, ne, xk, xv);
                    if (act && blk == bl) c = q0 + below;
                    pending &= ~__ballot_sync(0xffffffffu, act && blk == bl);
                }
            } else if (act) {
                const uint32_t q0 = blk * kSampleStride;
                uint32_t lo = 0, hi = min((uint32_t)kSampleStride, nb - q0);
                while (lo < hi) {
                    const uint32_t mid = (lo + hi) >> 1;
                    const uint64_t bk = __ldcg(p.d.sk + b0 + q0 + mid);
                    const bool lt = bk < xk || (bk == xk && __ldcg(p.d.sv + b0 + q0 + mid) < xv);
                    if (lt) lo = mid + 1; else hi = mid;
                }
                c = q0 + lo;
            }
            cnt += c;
        }
        s_cnt[warp][lane] = cnt;
        __syncthreads();
#ifndef MEDUSA_RANK_WARP_BLK
#define MEDUSA_RANK_WARP_BLK 1
#endif
        const uint32_t has_lanes = __ballot_sync(0xffffffffu, has);  // (every warp; used by warp 0)
        if (warp == 0 && has) {
            uint32_t rank = g - ta * kIsortTile;  // index inside its own tile
#pragma unroll
            for (int w = 0; w < kWarps; ++w) rank += s_cnt[w][lane];
            // (ordered compaction: a warp's keys take consecutive ranks, one or two
            // blocks; otherwise their ranks scatter and the combining only costs)
            if (MEDUSA_RANK_WARP_BLK && p.ordered) write_i_entry_warp(p, rank, nI, xv, ld_alloc(p.a.alloc + xv), has_lanes);
            else write_i_entry(p, rank, nI, xv, ld_alloc(p.a.alloc + xv));
        }
        __syncthreads();  // s_cnt is rewritten by the next range
    }
    pdl_trigger();
    TL_REC(3, 0, tl0);
}

// four sorted I bases (one 32-byte block, one L2 sector) in one load
__device__ __forceinline__ void ld_base4(const uint64_t* q, uint64_t& b0, uint64_t& b1, uint64_t& b2, uint64_t& b3) {
    asm volatile("ld.global.v4.u64 {%0, %1, %2, %3}, [%4];" : "=l"(b0), "=l"(b1), "=l"(b2), "=l"(b3) : "l"(q));
}

// count of sorted I bases <= x: the fences in shared memory, then the group of
// stride bases after the last fence <= x in 32-byte blocks (one sector each; 8-byte
// loads cost one sector per base: 2.5 us of k_iresolve's 7 us per CTA, measured)
// (fence: shared memory in k_iresolve, global in k_check_mi)
__device__ __forceinline__ uint32_t i_count_le(const uint64_t* fence, uint32_t nf, uint32_t stride, uint32_t nI,
                                               const uint64_t* i_base, uint64_t x) {
    uint32_t lo = 0;  // #{fences <= x}: binary lifting, no data-dependent branches
#pragma unroll
    for (uint32_t st = kFenceCap; st > 0; st >>= 1) {  // (reaches 2 kFenceCap - 1 >= nf)
        const uint32_t k = lo + st;
        if (k <= nf) lo = fence[k - 1] <= x ? k : lo;
    }
    if (lo == 0) return 0;
    const uint32_t g0 = (lo - 1) * stride, g1 = min(g0 + stride, nI);
    MCHECK(g0 < nI);
    uint32_t c = g0 + 1;  // base g0 (the fence) <= x
    for (uint32_t k = g0; k < g1; k += 8) {  // two blocks per round (a group of 4: one)
        uint64_t b[8];
        ld_base4(i_base + k, b[0], b[1], b[2], b[3]);
        if (k + 4 < g1) ld_base4(i_base + k + 4, b[4], b[5], b[6], b[7]);
        else b[4] = b[5] = b[6] = b[7] = ~0ull;
#pragma unroll
        for (int u = 0; u < 8; ++u) c += (k + u > g0 && k + u < g1 && b[u] <= x) ? 1u : 0u;
        if (b[7] > x) break;
    }
    return c;
}

// ----------------------------------------------------------------------------
// 4. k_classify: one CTA per 2048-word chunk.  The CTA sets up the chunk's
//    mortal window (registered mortals in list order, per-node live masks);
//    then each warp classifies its own 256 words with no further CTA barrier:
//    word q of warp w is q = 256 w + 32 k + lane (k = 0..7).
constexpr int kFront = 128;  // tree-query frontier nodes held per level (ALL10: <= 29)
struct ClsShared {
    uint64_t words[MEDUSA_CHUNK_WORDS];  // TMA destination; hit words then hold their record
    ulonglong2 rbe[kWinCap];             // (base, end) of one batch of window entries
    uint32_t rta[kWinCap], rtf[kWinCap], rid[kWinCap];
    uint64_t hmin[kWinCap / 32], hmax[kWinCap / 32];  // per loading warp: least base, greatest end
    uint32_t live[kNodeGrp][kWinCap / 32];  // live[u] bit e: window entry e live at node g0 + u
    // Segments: segment s of the chunk = the words of the s-th distinct node start
    // (segment 0 = node jf's words); s(q) = nsp[q/32] + popc(nsm[q/32] & bits 0..q%32)
    uint32_t nsm[MEDUSA_CHUNK_WORDS / 32];  // bit q: a node starts at word q (q > 0)
    uint32_t nsp[MEDUSA_CHUNK_WORDS / 32];  // exclusive popcount prefix of nsm
    uint32_t nt0[kNodeGrp];                 // launch positions of segments 0 .. kNodeGrp-1
    uint16_t cq[MEDUSA_CHUNK_WORDS];        // per warp (256 each): its candidates (word in chunk)
    uint32_t hits[MEDUSA_CHUNK_WORDS / 32]; // slot bits (warp w: words 8w .. 8w+7)
    uint32_t qbits[MEDUSA_CHUNK_WORDS / 32];// queued-candidate bits (same layout)

    uint64_t hull_lo, hull_hi;              // [least base, greatest end) of the current window batch
    union {
        uint32_t front[2][kFront];          // tree-query frontier (by level parity)
        uint32_t nt[kNodeGrp];              // launch positions of segments g0 .. g0+kNodeGrp-1 (later groups;
                                            //  used between queries only)
    };
    uint32_t fn[kMaxLevels + 1];            // frontier size per level
    uint32_t wid[kWinCap];                  // tree-query results: the window entries' allocation ordinals
    uint32_t nres;
    unsigned long long mbar;
};

#ifndef MEDUSA_CLS_SMEM
#define MEDUSA_CLS_SMEM 33792
#endif
// k_classify's dynamic shared memory: the window state (26 KB) padded to 33 KB, so
// that 6 classify CTAs fit on an SM (228 KB) instead of 8: the CTAs k_classify
// launches early (PDL) then leave room for the rank branch, which otherwise waits
// for classify CTAs to finish (k_rank started 6 us later, step span +2 us)
constexpr size_t kClsSmem = MEDUSA_CLS_SMEM > sizeof(ClsShared) ? MEDUSA_CLS_SMEM : sizeof(ClsShared);

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

// threads 0..kWinCap-1 (whole warps): the records of the m <= kWinCap window
// entries the tree query found -> S.r*, and each loading warp's least base /
// greatest end (the batch's hull)
__device__ __forceinline__ void window_load(const P& p, ClsShared& S, uint32_t m) {
    const uint32_t e = threadIdx.x;
    uint64_t b = ~0ull, en = 0;
    if (e < m) {
        const uint32_t id = S.wid[e];
        const medusa_alloc x = ld_alloc(p.a.alloc + id);
        S.rbe[e] = make_ulonglong2(x.base, x.base + x.size);
        S.rta[e] = x.t_alloc;
        S.rtf[e] = x.t_free;
        S.rid[e] = id;
        b = x.base;
        en = x.base + x.size;
    }
    b = warp_min_u64(b);
    en = warp_max_u64(en);
    if ((e & 31) == 0) {
        S.hmin[e >> 5] = b;
        S.hmax[e >> 5] = en;
    }
}

// CTA-wide descent of the mortal tree: the window entries of the
// chunk = the ordinals i in [o_lo, o_hi) with v_i > T0 (a mortal freed after the
// chunk's first launch) and t_alloc_i < T1 (allocated before its last launch)
// and, when every segment's launch position is in nt0 (exact), live at one of
// them: t_alloc_i < nt0[u] < t_free_i for some u.  The descent starts at the
// highest level with <= kThreads nodes (one thread each: q_seed) and goes one
// level per round (q_expand: each warp expands one kept node into its 32
// children with one coalesced load).  Kept nodes of level l go to
// S.front[l & 1], the entries (level 0) to S.wid[0 .. S.nres).
struct QRange {
    uint32_t T0, T1, o_lo, o_hi, ng0;
    bool exact;
};

__device__ __forceinline__ int q_start(const Tree& T) { return T.l0; }

// #{u < n : a[u] <= y} (kStrict: a[u] < y) of an ascending array of n < 2 kTop
// entries in shared memory: binary lifting, no data-dependent branches
template <uint32_t kTop, bool kStrict = false>
__device__ __forceinline__ uint32_t count_upto(const uint32_t* a, uint32_t n, uint32_t y) {
    uint32_t c = 0;
#pragma unroll
    for (uint32_t st = kTop; st > 0; st >>= 1) {
        const uint32_t k = c + st;  // take a[c .. k) if it is in range and its last entry qualifies
        if (k <= n) c = (kStrict ? a[k - 1] < y : a[k - 1] <= y) ? k : c;
    }
    return c;
}

__device__ __forceinline__ bool q_test(const Tree& T, const ClsShared& S, int l, uint32_t c, const QRange& q) {
    if (c >= T.cnt[l]) return false;
    const uint32_t sh = 5u * (uint32_t)l;  // a node of level l covers 2^sh ordinals
    const uint64_t first = (uint64_t)c << sh, last = first + (1ull << sh);
    if (!(first < q.o_hi && last > q.o_lo)) return false;
    const uint2 nd = l > 0 ? __ldcg(T.node + T.off[l] + c) : __ldcg(T.leaf + c);
    bool keep = nd.x > q.T0 && nd.y < q.T1;
    if (keep && l == 0 && q.exact) {  // live at one of the chunk's launches
        const uint32_t lo = count_upto<kNodeGrp>(S.nt0, q.ng0, nd.y);  // the first segment launched after t_alloc
        MCHECK(lo <= q.ng0 && q.ng0 <= (uint32_t)kNodeGrp);
        keep = lo < q.ng0 && S.nt0[lo] < nd.x;
    }
    return keep;
}

// (whole warp) appends the lanes' kept nodes of level l; false if the list overflows
__device__ __forceinline__ bool q_push(ClsShared& S, int l, bool keep, uint32_t c) {
    const uint32_t b = __ballot_sync(0xffffffffu, keep);
    if (!b) return true;
    const uint32_t lane = threadIdx.x & 31;
    uint32_t* out = l > 0 ? S.front[l & 1] : S.wid;
    uint32_t* cnt = l > 0 ? &S.fn[l] : &S.nres;
    const uint32_t cap = l > 0 ? (uint32_t)kFront : (uint32_t)kWinCap;
    uint32_t base = 0;
    if (lane == 0) base = atomicAdd(cnt, (uint32_t)__popc(b));
    base = __shfl_sync(0xffffffffu, base, 0);
    const uint32_t pos = base + __popc(b & lanemask_lt());
    if (keep && pos < cap) out[pos] = c;
    return !(keep && pos >= cap);
}

// (whole CTA, no barrier) the start level's nodes, one per thread
__device__ __forceinline__ bool q_seed(const Tree& T, ClsShared& S, int l, const QRange& q) {
    const uint32_t c = threadIdx.x;
    return q_push(S, l, q_test(T, S, l, c, q), c);
}

// (whole CTA, no barrier) the children at level l of the kept nodes of level l+1
__device__ __forceinline__ bool q_expand(const Tree& T, ClsShared& S, int l, const QRange& q) {
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t np = min(S.fn[l + 1], (uint32_t)kFront);
    const uint32_t* par = S.front[(l + 1) & 1];
    bool ok = true;
    for (uint32_t f = warp; f < np; f += kWarps) {
        const uint32_t c = par[f] * 32 + lane;
        ok &= q_push(S, l, q_test(T, S, l, c, q), c);
    }
    return ok;
}

// (whole CTA) counters of a query; the caller's next barrier publishes them
__device__ __forceinline__ void q_reset(ClsShared& S) {
    if (threadIdx.x <= (uint32_t)kMaxLevels) S.fn[threadIdx.x] = 0;
    if (threadIdx.x == 0) S.nres = 0;
}

// a whole query over [q.o_lo, q.o_hi); false on overflow (the caller halves the range)
__device__ bool tree_query(const Tree& T, ClsShared& S, const QRange& q) {
    q_reset(S);
    __syncthreads();
    const int l0 = q_start(T);
    if (__syncthreads_or(!q_seed(T, S, l0, q))) return false;
    for (int l = l0 - 1; l >= 0; --l)
        if (__syncthreads_or(!q_expand(T, S, l, q))) return false;
    return true;
}

// The live masks of nodes g0 .. g0+ng for the loaded batch of m entries (whole CTA;
// nt = their launch positions).  Entry e is live at nodes u0 <= u < u1
// (t_alloc < t_u < t_free): toggle bit e at u0 and u1, then a prefix XOR over u.
// (cleared: the live masks were zeroed before the caller's last barrier)
__device__ __forceinline__ void build_live(ClsShared& S, const uint32_t* nt, uint32_t ng, uint32_t m, bool cleared) {
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {  // the batch's address hull
        uint64_t lo = ~0ull, hi = 0;
        for (uint32_t w = 0; w < (m + 31) / 32; ++w) { lo = min(lo, S.hmin[w]); hi = max(hi, S.hmax[w]); }
        S.hull_lo = lo;
        S.hull_hi = hi;
    }
    if (!cleared) {
        for (uint32_t k = tid; k < kNodeGrp * (kWinCap / 32); k += kThreads) (&S.live[0][0])[k] = 0u;
        __syncthreads();
    }
    for (uint32_t e = tid; e < m; e += kThreads) {
        const uint32_t ta = S.rta[e], tf = S.rtf[e];
        const uint32_t u0 = count_upto<kNodeGrp>(nt, ng, ta);        // #{u : t_u <= t_alloc}
        const uint32_t u1 = count_upto<kNodeGrp, true>(nt, ng, tf);  // #{u : t_u < t_free}
        if (u0 < u1) {
            atomicXor(&S.live[u0][e >> 5], 1u << (e & 31));
            if (u1 < ng) atomicXor(&S.live[u1][e >> 5], 1u << (e & 31));
        }
    }
    __syncthreads();
    static_assert(kNodeGrp == 128, "prefix XOR: 4 nodes per lane");
    for (uint32_t w = warp; w < (m + 31) / 32; w += kWarps) {  // one warp per mask word
        uint32_t v[4], run = 0;
#pragma unroll
        for (int r = 0; r < 4; ++r) { v[r] = S.live[lane * 4 + r][w]; run ^= v[r]; v[r] = run; }
        uint32_t incl = run;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= (uint32_t)d) incl ^= y;
        }
        const uint32_t before = incl ^ run;
#pragma unroll
        for (int r = 0; r < 4; ++r) S.live[lane * 4 + r][w] = v[r] ^ before;
    }
    __syncthreads();
}

// The window entry holding word x at node u - g0 of the current group, or -1:
// the live entries of one launch are pairwise disjoint (a well-formed trace), so
// the first live entry whose range holds x is the only one.
__device__ __forceinline__ int window_find(const ClsShared& S, uint32_t m, uint32_t ul, uint64_t x) {
    if (x < S.hull_lo || x >= S.hull_hi) return -1;
    // the entries live at the node (a handful: ~4 mortals are live at a launch in
    // the BASELINE sets) -- at most one holds x.  32-bit shared-window addresses
    // (ld.shared): no generic-to-shared base rebuilt inside the loop
    const uint32_t a_live = smem_u32(&S.live[ul][0]), a_rbe = smem_u32(S.rbe);
    for (uint32_t w = 0; w < (m + 31) / 32; ++w) {
        uint32_t bits;
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(bits) : "r"(a_live + 4 * w));
        while (bits) {
            const uint32_t e = w * 32 + __ffs(bits) - 1;
            bits &= bits - 1;
            uint64_t b, en;  // one 16-byte load of (base, end)
            asm volatile("ld.shared.v2.u64 {%0, %1}, [%2];" : "=l"(b), "=l"(en) : "r"(a_rbe + 16 * e));
            if (b <= x && x < en) { MCHECK(e < m); return (int)e; }
        }
    }
    return -1;
}

// segment (see ClsShared) of word q of the chunk
__device__ __forceinline__ uint32_t seg_of(const ClsShared& S, uint32_t q) {
    return S.nsp[q >> 5] + __popc(S.nsm[q >> 5] & (0xFFFFFFFFu >> (31 - (q & 31))));
}

// launch position of the node holding word q (segments beyond group 0: search node_off)
__device__ __forceinline__ uint32_t seg_time(const P& p, const ClsShared& S, uint32_t s, uint64_t g, uint32_t jf,
                                             uint32_t jl) {
    if (s < kNodeGrp) return S.nt0[s];
    uint32_t lo = jf + 1, hi = jl + 1;  // first node starting after word g
    while (lo < hi) { const uint32_t mid = (lo + hi) >> 1; if (p.a.node_off[mid] <= g) lo = mid + 1; else hi = mid; }
    return __ldg(p.a.node_t + lo - 1);
}

// launch positions of segments g0 .. g0+ng-1 into nt (whole CTA; nt zeroed here)
__device__ __forceinline__ void seg_times(const P& p, ClsShared& S, uint32_t* nt, uint32_t g0, uint32_t ng, uint64_t cs,
                                          uint32_t jf, uint32_t jl) {
    for (uint32_t u = threadIdx.x; u < ng; u += kThreads) nt[u] = 0;
    __syncthreads();
    if (threadIdx.x == 0 && g0 == 0) nt[0] = p.a.node_t[jf];
    for (uint32_t j = jf + 1 + threadIdx.x; j <= jl; j += kThreads) {
        const uint32_t q = (uint32_t)(p.a.node_off[j] - cs);
        if (q >= kChunkWords) continue;
        const uint32_t s = seg_of(S, q);
        if (s >= g0 && s < g0 + ng) atomicMax(nt + (s - g0), p.a.node_t[j]);  // the last node of a start is its non-empty one
    }
    __syncthreads();
}

__device__ void classify_role(const P& p, uint32_t c, ClsShared& S) {
    const MaterializeArgs& a = p.a;
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const Ctl* ctl = p.d.ctl;
    unsigned long long tl_p = TL_NOW();
    const uint64_t cs = (uint64_t)c * kChunkWords;
    const uint32_t n = (uint32_t)min((uint64_t)kChunkWords, a.n_words - cs);
    const uint64_t* gsrc = a.words + cs;
    const bool tma = ((reinterpret_cast<uintptr_t>(gsrc) & 15) == 0) && (n % 2 == 0);
    const uint32_t mb = smem_u32(&S.mbar);
    // A. the chunk's words -> shared memory with one TMA bulk copy, issued before
    //    waiting for k_trace (the words are an input; k_trace lets this grid start
    //    at once in the slots it leaves free)
    if (tid == 0 && tma) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(n * 8) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(smem_u32(S.words)), "l"(gsrc), "r"(n * 8), "r"(mb) : "memory");
    }
    if (tid < MEDUSA_CHUNK_WORDS / 32) S.nsm[tid] = 0;
    if (tid < kNodeGrp) S.nt0[tid] = 0;
    q_reset(S);
    pdl_wait();  // k_trace: node ranges, status, prefilter bounds, the mortal tree
    // every value this CTA needs from k_trace, loaded in one round (the node
    // range is read before the status is known; it is used only if valid)
    const uint32_t N = a.n_nodes;
    const uint32_t st = __ldcg(&ctl->status);
    const uint2 jf2 = N ? __ldcg(p.d.jf + c) : make_uint2(0, 0), jl2 = N ? __ldcg(p.d.jl + c) : make_uint2(0, 0);
    const uint64_t gmin = ~__ldcg(&ctl->gmin_c), gmax = __ldcg(&ctl->gmax);
    // A malformed CSR or launch order (flagged by k_trace) leaves jf / jl and the
    // node offsets meaningless: write the empty counts the later kernels read and
    // do nothing else (the call returns INVALID_ARG; no shared-memory index is
    // ever derived from node_off); the bulk copy is waited for before leaving
    if (st & ST_INVALID) {
        if (tid < kWarps) p.d.qcnt[c * kWarps + tid] = 0;
        if (tid == 0 && tma) {
            uint32_t done = 0;
            while (!done) {
                asm volatile("{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], 0; selp.u32 %0, 1, 0, P; }"
                             : "=r"(done) : "r"(mb) : "memory");
            }
        }
        pdl_trigger();
        return;
    }
    const uint32_t jf = N ? min(jf2.x, N - 1) : 0, jl = N ? min(jl2.x, N - 1) : 0;
    const uint32_t t_jf = jf2.y, t_jl = jl2.y;  // the chunk's first and last launch positions
    const uint32_t nn = N ? jl - jf + 1 : 0;
    if (!tma)
        for (uint32_t q = tid; q < n; q += kThreads) S.words[q] = ld_stream(gsrc + q);
    const uint32_t n_alloc = a.n_alloc;
    const bool use_tree = N && n_alloc;
    const Tree& T = p.d.tree;
    const int l0 = q_start(T);
    QRange qr{t_jf, t_jl, 0u, n_alloc, 0u, true};
    __syncthreads();  // nsm / nt0 / query counters zeroed before any thread sets them
    TL_PHASE(4, 10, tl_p);  // A: setup
    // B. the starts of the chunk's nodes (-> start bitmask, its popcount prefix,
    //    the launch positions of the first kNodeGrp segments), interleaved with
    //    the first two rounds of the window's tree query (the internal levels
    //    need only the chunk's first and last launch positions)
    bool qok = true;
    if (use_tree && l0 >= 1) qok &= q_seed(T, S, l0, qr);
    uint32_t my_q = 0xFFFFFFFFu, my_t = 0;  // this thread's first node (start, launch position)
    for (uint32_t j = jf + 1 + tid; j <= jl; j += kThreads) {
        const uint32_t q = (uint32_t)(a.node_off[j] - cs);
        if (q >= n) continue;  // (a valid CSR puts every start of (jf, jl] inside the chunk)
        if (my_q == 0xFFFFFFFFu) { my_q = q; my_t = a.node_t[j]; }
        atomicOr(&S.nsm[q >> 5], 1u << (q & 31));
    }
    __syncthreads();
    if (warp == 1) {  // exclusive popcount prefix of the 64 start-mask words
        const uint32_t c0 = __popc(S.nsm[2 * lane]), c1 = __popc(S.nsm[2 * lane + 1]);
        uint32_t incl = c0 + c1;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= (uint32_t)d) incl += y;
        }
        S.nsp[2 * lane] = incl - c0 - c1;
        S.nsp[2 * lane + 1] = incl - c1;
    }
    if (use_tree && l0 >= 2) qok &= q_expand(T, S, l0 - 1, qr);
    __syncthreads();
    const uint32_t n_seg = N ? S.nsp[63] + __popc(S.nsm[63]) + 1 : 0;
    const uint32_t ng0 = min((uint32_t)kNodeGrp, n_seg);
    qr.ng0 = ng0;
    qr.exact = n_seg <= (uint32_t)kNodeGrp;
    // launch positions of segments 0..ng0-1 (the last node of a start is its non-empty one)
    if (tid == 0 && N) atomicMax(&S.nt0[0], t_jf);
    if (my_q != 0xFFFFFFFFu) {
        const uint32_t sg = seg_of(S, my_q);
        if (sg < kNodeGrp) atomicMax(&S.nt0[sg], my_t);
    }
    if (nn > (uint32_t)kThreads + 1) {  // more nodes than threads: the rest
        for (uint32_t j = jf + 1 + kThreads + tid; j <= jl; j += kThreads) {
            const uint32_t q = (uint32_t)(a.node_off[j] - cs);
            if (q >= n) continue;
            const uint32_t sg = seg_of(S, q);
            if (sg < kNodeGrp) atomicMax(&S.nt0[sg], a.node_t[j]);
        }
    }
    // C. this warp's words: candidates (inside [least base, greatest end) of the
    //    trace) compacted into the warp's list
    if (tma) {
        uint32_t done = 0;
        while (!done) {
            asm volatile("{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], 0; selp.u32 %0, 1, 0, P; }"
                         : "=r"(done) : "r"(mb) : "memory");
        }
    }
    uint16_t* wl = S.cq + warp * 256;   // this warp's candidates (word in chunk)
    uint32_t* wh = S.hits + warp * 8;   // hit bits of the warp's 256 words
    uint32_t nc = 0;
    const uint32_t lt = lanemask_lt();
#pragma unroll
    for (int k = 0; k < kWordsPerThread / 2; ++k) {  // two words per lane: one 16-B shared load
        const uint32_t q = warp * 256 + k * 64 + 2 * lane;
        const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(&S.words[q]);
        const bool c0 = q < n && v.x >= gmin && v.x < gmax;
        const bool c1 = q + 1 < n && v.y >= gmin && v.y < gmax;
        const uint32_t b0 = __ballot_sync(0xffffffffu, c0), b1 = __ballot_sync(0xffffffffu, c1);
        uint32_t o = nc + __popc(b0 & lt) + __popc(b1 & lt);  // ascending word order
        if (c0) wl[o++] = (uint16_t)q;
        if (c1) wl[o] = (uint16_t)(q + 1);
        nc += __popc(b0) + __popc(b1);
    }
    if (lane < 8) { wh[lane] = 0; S.qbits[warp * 8 + lane] = 0; }
    // the rest of the query (the leaves need nt0: complete after this barrier)
    qok = !__syncthreads_or(!qok);
    TL_PHASE(4, 11, tl_p);  // B/C: node starts, TMA wait, candidates, upper query levels
    if (use_tree && qok) {
        for (int l = l0 >= 2 ? l0 - 2 : 0; l >= 0; --l) {
            if (l == l0) qok = !__syncthreads_or(!q_seed(T, S, l, qr));  // (l0 == 0: the leaves are the start level)
            else qok = !__syncthreads_or(!q_expand(T, S, l, qr));
            if (!qok) break;
        }
    }
    // D. the window: the mortals live at one of the chunk's launches (normally one
    //    batch of <= kWinCap entries; a query that overflows is retried on half the
    //    ordinal range, and the ranges are then processed one batch after
    //    another).  Per batch and node group (normally one: <= kNodeGrp
    //    segments): the live masks, then each warp looks its own candidates up
    //    among the entries live at their node.
    bool have = qok;  // results of the first query (the whole ordinal range) in S.wid
    uint32_t o_lo = 0, wlen = qok ? n_alloc : (n_alloc + 1) / 2;
    while (use_tree && o_lo < n_alloc) {
        uint32_t o_hi = n_alloc;
        if (!have) {
            o_hi = (uint32_t)min((uint64_t)o_lo + wlen, (uint64_t)n_alloc);
            qr.o_lo = o_lo;
            qr.o_hi = o_hi;
            if (!tree_query(T, S, qr)) {
                wlen = (wlen + 1) / 2;
                continue;
            }
        }
        have = false;
        const uint32_t m = S.nres;
        if (o_hi < n_alloc) __syncthreads();  // every thread has read nres before a later query resets it
        TL_PHASE(4, 12, tl_p);  // D: tree query
        if (m) {
            if (tid < kWinCap) window_load(p, S, m);
            else  // the other threads zero the live masks meanwhile (the first group's)
                for (uint32_t k = tid - kWinCap; k < kNodeGrp * (kWinCap / 32); k += kThreads - kWinCap)
                    (&S.live[0][0])[k] = 0u;
            __syncthreads();
            for (uint32_t g0 = 0; g0 < n_seg; g0 += kNodeGrp) {
                const uint32_t ng = min((uint32_t)kNodeGrp, n_seg - g0);
                const uint32_t* nt = S.nt0;
                if (g0) {
                    seg_times(p, S, S.nt, g0, ng, cs, jf, jl);
                    nt = S.nt;
                }
                build_live(S, nt, ng, m, g0 == 0);
                for (uint32_t i = lane; i < nc; i += 32) {
                    const uint32_t q = wl[i];
                    if ((wh[(q & 255) >> 5] >> (q & 31)) & 1u) continue;  // found in an earlier batch
                    const uint32_t u = seg_of(S, q);
                    if (u < g0 || u >= g0 + ng) continue;
                    const uint64_t x = S.words[q];
                    const int e = window_find(S, m, u - g0, x);
                    if (e >= 0) {
                        S.words[q] = ((uint64_t)S.rid[e] << MEDUSA_OFF_BITS) | (x - S.rbe[e].x);
                        atomicOr(&wh[(q & 255) >> 5], 1u << (q & 31));
                    }
                }
                // the live masks / window are rewritten by the next group / batch; after
                // the last one each warp goes on to its own records (nothing it reads there
                // is rewritten), so a warp with few lookups does not wait for the others
#ifndef MEDUSA_CLS_LAST_BARRIER
#define MEDUSA_CLS_LAST_BARRIER 0
#endif
                if (MEDUSA_CLS_LAST_BARRIER || !(g0 + kNodeGrp >= n_seg && o_hi >= n_alloc)) __syncthreads();
            }
        }
        TL_PHASE(4, 13, tl_p);  // D: live masks, window search
        o_lo = o_hi;
        wlen = (uint32_t)min((uint64_t)wlen * 2, (uint64_t)n_alloc);
    }
    // E. the warp's candidates: window hits (records in S.words) and the rest,
    //    queued for the I-list search, written to the warp's record and queue
    //    regions in word order; no CTA barrier: every warp finishes on its own
    {
        uint32_t* wqb = S.qbits + warp * 8;
        const uint32_t region = (c * kWarps + warp) * p.d.cap_pw, cap = p.d.cap_pw;
        const uint32_t lt = lanemask_lt();
        uint32_t kr = 0, kq = 0;
        for (uint32_t i0 = 0; i0 < nc; i0 += 32) {
            const uint32_t i = i0 + lane;
            bool hit = false, need = false;
            uint32_t q = 0;
            if (i < nc) {
                q = wl[i];
                hit = (wh[(q & 255) >> 5] >> (q & 31)) & 1u;
                need = !hit;
            }
            const uint32_t bh = __ballot_sync(0xffffffffu, hit), bn = __ballot_sync(0xffffffffu, need);
            if (hit) {
                const uint32_t k = kr + __popc(bh & lt);
                if (k < cap) p.d.rec[region + k] = S.words[q];
            } else if (need) {
                const uint32_t k = kq + __popc(bn & lt);
                const uint32_t t = seg_time(p, S, seg_of(S, q), cs + q, jf, jl);  // the word's launch position
                if (k < cap) p.d.queue[region + k] = IQ{S.words[q], (uint32_t)(cs + q), t};
                atomicOr(&wqb[(q & 255) >> 5], 1u << (q & 31));
            }
            kr += __popc(bh);
            kq += __popc(bn);
        }
        if (max(kr, kq) > cap) {  // the warp's regions are too small: rerun with whole-warp ones
            if (lane == 0) {
                atomicMax(&p.d.ctl->need_pw, max(kr, kq));
                flag(p.d.ctl, ST_OVERFLOW);
            }
            kq = min(kq, cap);
        }
        __syncwarp();
        const uint64_t n_mask = (a.n_words + 31) / 32;
        if (lane < 8) {  // the warp's 8 mask words, one lane each
            const uint32_t qw = warp * 256 + lane * 32;
            const uint64_t mw = (cs + qw) >> 5;
            if (qw < n && mw < n_mask) {
                a.mask[mw] = wh[lane];
                p.d.imask[mw] = 0;
                p.d.qmask[mw] = wqb[lane];
            }
        }
        if (lane == 0) {
            p.d.qcnt[c * kWarps + warp] = kq;
            // the chunk's slot count (k_iresolve adds the I-list slots; k_emit turns
            // the counts into chunk_base) and its 256-chunk group sum
            if (kr) {
                atomicAdd(p.d.chunk_cnt + c, kr);
                atomicAdd(p.d.chunk_sup + (c >> 8), (unsigned long long)kr);
            }
        }
    }
    TL_PHASE(4, 15, tl_p);  // E: records, queue, mask words
    pdl_trigger();
}

// ----------------------------------------------------------------------------
// 2c. The R-Q7 checks (default priority; they only set ST_TRACE), per warp a
//     block of 32 allocation ordinals, one per lane ("mine" = a mortal):
//     k_check_mm (after k_trace): M-M -- each mortal j against the mortals
//       i < j still live when j is allocated (t_free_i > t_alloc_j), found by a
//       depth-first descent of the mortal tree (nodes with max t_free > the
//       block's least t_alloc and first ordinal < its greatest ordinal), then
//       hull-filtered and tested pairwise;
//     k_check_mi (after k_rank): I-I -- adjacent sorted I entries; M-I -- each
//       mortal against the run of I entries its range meets (one fence search;
//       the common "no I entry in range" case costs two more loads).
constexpr int kStk = 32 * kMaxLevels + 32;  // DFS stack per warp: < 32 entries per level on the path

// this lane's allocation of block b and whether it is a mortal
__device__ __forceinline__ bool check_mine(const P& p, uint32_t j, medusa_alloc& x, uint32_t& t_last) {
    const uint32_t N = p.a.n_nodes;
    t_last = N ? p.a.node_t[N - 1] : 0;
    x = medusa_alloc{};
    if (j >= p.a.n_alloc) return false;
    x = ld_alloc(p.a.alloc + j);
    return x.size != 0 && !(N && x.t_alloc < t_last && t_last < x.t_free);
}

__global__ void __launch_bounds__(kThreads) k_check_mm(P p) {
    __shared__ ulonglong2 s_be[kWarps][32];  // (base, end): one 16-byte broadcast load
    __shared__ uint2 s_ti[kWarps][32];       // (t_free, id): one 8-byte broadcast load
    __shared__ uint32_t s_stk[kWarps][kStk];
    const unsigned long long tl0 = TL_NOW();
    const Tree& T = p.d.tree;
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t b = blockIdx.x * kWarps + warp;
    if (b >= p.nb) return;  // whole warp
    const uint32_t j = b * 32 + lane;
    medusa_alloc x;
    uint32_t t_last;
    const bool mine = check_mine(p, j, x, t_last);
    const uint64_t xe = x.base + x.size;
    bool bad = false;
    const uint64_t hb = warp_min_u64(mine ? x.base : ~0ull), he = warp_max_u64(mine ? xe : 0ull);
    const uint32_t hta = __reduce_min_sync(0xffffffffu, mine ? x.t_alloc : 0xFFFFFFFFu);
    const uint32_t hj = __reduce_max_sync(0xffffffffu, mine ? j : 0u);
    if (he) {
        uint32_t* stk = s_stk[warp];
        uint32_t sp = 0;
        int lvl = (int)T.top + 1;  // the virtual root: its children are the top level
        uint32_t node = 0;
        while (true) {
            const int cl = lvl - 1;  // level of the children
            const uint32_t c = node * 32 + lane;
            const uint32_t sh = 5u * (uint32_t)cl;
            bool keep = false;
            uint2 nd = make_uint2(0, 0);
            ulonglong2 be = make_ulonglong2(0, 0);
            if (c < T.cnt[cl] && ((uint64_t)c << sh) < hj) {
                nd = cl > 0 ? __ldcg(T.node + T.off[cl] + c) : __ldcg(T.leaf + c);
                if (cl == 0) be = __ldcg(T.leaf_be + c);  // (same round)
                keep = nd.x > hta;
            }
            const uint32_t kb = __ballot_sync(0xffffffffu, keep);
            if (cl > 0) {  // push the kept children (the stack holds (level << 24) | node)
                if (keep) stk[sp + __popc(kb & lanemask_lt())] = ((uint32_t)cl << 24) | c;
                sp += __popc(kb);
            } else if (kb) {  // leaves: mortals i < hj with t_free_i > hta
                const uint64_t yb = be.x, ye = be.y;
                const bool k2 = keep && yb < he && hb < ye;
                const uint32_t k2b = __ballot_sync(0xffffffffu, k2);
                __syncwarp();
                if (k2) {
                    const uint32_t o = __popc(k2b & lanemask_lt());
                    s_be[warp][o] = make_ulonglong2(yb, ye);
                    s_ti[warp][o] = make_uint2(nd.x, c);  // (t_free, id)
                }
                __syncwarp();
                if (mine) {
                    const uint32_t nk = __popc(k2b);
                    for (uint32_t q = 0; q < nk; ++q) {
                        const ulonglong2 be = s_be[warp][q];
                        const uint2 ti = s_ti[warp][q];
                        bad |= (ti.y < j) & (ti.x > x.t_alloc) & (be.x < xe) & (x.base < be.y);
                    }
                }
            }
            __syncwarp();
            if (sp == 0) break;
            const uint32_t e = stk[--sp];
            __syncwarp();  // every lane has read the popped entry before the next push reuses its slot
            lvl = (int)(e >> 24);
            node = e & 0xFFFFFFu;
        }
    }
    if (bad) flag(p.d.ctl, ST_TRACE);
    TL_REC(8, 0, tl0);
}

__global__ void __launch_bounds__(kThreads) k_check_mi(P p) {
    const unsigned long long tl0 = TL_NOW();
    const uint32_t cta = blockIdx.x;
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t nI = p.d.ctl->nI;
    {  // I-I: sorted neighbours must not overlap (all of I is live at the last launch)
        const uint32_t k = cta * blockDim.x + threadIdx.x;
        if (k + 1 < nI && p.d.i_rest[k].end > p.d.i_base[k + 1]) flag(p.d.ctl, ST_TRACE);
    }
    const uint32_t stride = fence_stride(nI);
    const uint32_t nf = (nI + stride - 1) / stride;
    const uint32_t b = cta * kWarps + warp;
    if (b >= p.nb) return;  // whole warp
    const uint32_t j = b * 32 + lane;
    medusa_alloc x;
    uint32_t t_last;
    const bool mine = check_mine(p, j, x, t_last);
    const uint64_t xe = x.base + x.size;
    bool bad = false;
    // M-I: the I entries meeting [base, end) are one run [s, e) of the sorted list
    if (mine && nI) {
        const uint32_t k0 = i_count_le(p.d.fence, nf, stride, nI, p.d.i_base, x.base);  // bases <= base
        const uint32_t s = (k0 > 0 && p.d.i_rest[k0 - 1].end > x.base) ? k0 - 1 : k0;
        uint32_t e = k0;  // bases < end
        if (k0 < nI && p.d.i_base[k0] < xe) e = i_count_le(p.d.fence, nf, stride, nI, p.d.i_base, xe - 1);
        // overlap with I entry e: m freed before T_last -> t_alloc_e < t_free_m; else t_free_e > t_alloc_m
        const bool freed_early = x.t_free <= t_last;
        uint32_t k = s;
        for (; k < e && (k % kIBlk) != 0; ++k)
            bad |= freed_early ? p.d.i_rest[k].t_alloc < x.t_free : p.d.i_tf[k] > x.t_alloc;
        for (; k + kIBlk <= e; k += kIBlk)
            bad |= freed_early ? ~p.d.blk_min_ta_c[k / kIBlk] < x.t_free : p.d.blk_max_tf[k / kIBlk] > x.t_alloc;
        for (; k < e; ++k)
            bad |= freed_early ? p.d.i_rest[k].t_alloc < x.t_free : p.d.i_tf[k] > x.t_alloc;
    }
    if (bad) flag(p.d.ctl, ST_TRACE);
    TL_REC(9, 0, tl0);
}

#ifndef MEDUSA_CLS_MINB
#define MEDUSA_CLS_MINB 7  // classify CTAs per SM (shared memory allows 7)
#endif
__global__ void __launch_bounds__(kThreads, MEDUSA_CLS_MINB) k_classify(P p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    const unsigned long long tl0 = TL_NOW();
    classify_role(p, blockIdx.x, *reinterpret_cast<ClsShared*>(smem_raw));  // (waits for k_prepare inside)
    TL_REC(4, 0, tl0);
}

// ----------------------------------------------------------------------------
// 4b. k_iresolve (after k_rank and k_classify): the queued candidates against the
//     sorted I list.  Persistent CTAs loop over chunks, fences loaded once per
//     CTA before the wait for k_classify; the chunk's eight queue ranges (one per classify warp) are spread over
//     the whole CTA (entry i of their concatenation -> thread i mod 256: a long
//     range no longer sets the chunk's time; per-warp ranges measured ALL10
//     iresolve 16.0 vs 13.8 us span).  Per candidate one group of bases and one
//     entry (two dependent loads); a hit writes its record over its queue
//     entry's word and sets its bit in a shared copy of the chunk's I-resolved
//     bits, which go to the mask (one red.or per mask word) and the I-resolved
//     mask (one store per word) at the chunk's end; the chunk's count grows by
//     one atomic per warp.
#ifndef MEDUSA_IRES_SMEM_MASK
#define MEDUSA_IRES_SMEM_MASK 1  // a chunk's I-resolved bits gathered in shared memory, one atomic per mask word
#endif
__global__ void __launch_bounds__(kThreads, 6) k_iresolve(P p) {
    __shared__ uint64_t s_fence[kFenceCap];
    const unsigned long long tl0 = TL_NOW();
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // the sorted I list is complete when this grid starts (k_isort / k_rank are a
    // full dependency through the 'ranked' event, k_trace one before them): the
    // fences come in before the wait for k_classify
    const uint32_t nI = __ldcg(&p.d.ctl->nI);
    {
        const uint32_t stride = fence_stride(nI);
        const uint32_t nf = nI ? (nI + stride - 1) / stride : 0u;
        for (uint32_t f = tid; f < nf; f += kThreads) s_fence[f] = __ldcg(p.d.fence + f);
    }
    pdl_wait();  // k_classify: queue, counts, masks
    if (nI) {
        // the chunk's queue ranges (one per classify warp) taken by the whole CTA:
        // entry i of the chunk's concatenated ranges -> thread i mod 256, so a warp
        // whose range is long (up to cap_pw entries) does not set the chunk's time
        __shared__ uint32_t s_pre[kWarps + 1];
        __shared__ uint32_t s_mb[kChunkWords / 32];  // the chunk's I-resolved bits (MEDUSA_IRES_SMEM_MASK)
        const uint32_t stride = fence_stride(nI);
        const uint32_t nf = (nI + stride - 1) / stride;
        const uint32_t cap = p.d.cap_pw;
        uint32_t my_cnt = (blockIdx.x < p.C && tid < kWarps) ? min(__ldcg(p.d.qcnt + blockIdx.x * kWarps + tid), cap) : 0u;
        for (uint32_t c = blockIdx.x; c < p.C; c += gridDim.x) {
            if (warp == 0) {  // exclusive prefix of the 8 range lengths
                uint32_t incl = lane < kWarps ? my_cnt : 0u;
#pragma unroll
                for (int d = 1; d < kWarps; d <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                    if (lane >= (uint32_t)d) incl += y;
                }
                if (lane < kWarps) s_pre[lane + 1] = incl;
                if (lane == 0) s_pre[0] = 0;
            }
            if (MEDUSA_IRES_SMEM_MASK && tid < kChunkWords / 32) s_mb[tid] = 0;
            __syncthreads();  // (also: the fences, on the first chunk)
            const uint32_t cn = c + gridDim.x;  // the next chunk's counts, loaded early
            if (tid < kWarps) my_cnt = cn < p.C ? min(__ldcg(p.d.qcnt + cn * kWarps + tid), cap) : 0u;
            const uint32_t total = s_pre[kWarps];
            uint32_t cnt = 0;
            for (uint32_t i0 = 0; i0 < total; i0 += kThreads) {
                const uint32_t i = i0 + tid;
                bool hit = false;
                if (i < total) {
                    uint32_t w = 0;  // the range holding entry i
#pragma unroll
                    for (int r = 1; r < kWarps; ++r) w += s_pre[r] <= i ? 1u : 0u;
                    const uint64_t k = (uint64_t)(c * kWarps + w) * cap + (i - s_pre[w]);
                    const IQ q = p.d.queue[k];
                    const uint32_t le = i_count_le(s_fence, nf, stride, nI, p.d.i_base, q.x);
                    if (le) {
                        const uint64_t base = p.d.i_base[le - 1];
                        const IRest e = p.d.i_rest[le - 1];
                        if (q.x < e.end && e.t_alloc < q.t) {
                            hit = true;
                            p.d.queue[k].x = ((uint64_t)e.id << MEDUSA_OFF_BITS) | (q.x - base);
                            if (MEDUSA_IRES_SMEM_MASK) {
                                MCHECK(q.g >= c * kChunkWords && q.g - c * kChunkWords < (uint32_t)kChunkWords);
                                atomicOr(&s_mb[(q.g - c * kChunkWords) >> 5], 1u << (q.g & 31));
                            } else {
                                atomicOr(p.a.mask + (q.g >> 5), 1u << (q.g & 31));
                                atomicOr(p.d.imask + (q.g >> 5), 1u << (q.g & 31));
                            }
                        }
                    }
                }
                cnt += __popc(__ballot_sync(0xffffffffu, hit));
            }
            if (lane == 0 && cnt) {
                atomicAdd(p.d.chunk_cnt + c, cnt);
                atomicAdd(p.d.chunk_sup + (c >> 8), (unsigned long long)cnt);
            }
            if (MEDUSA_IRES_SMEM_MASK) {  // the chunk's bits: one reduction per mask word (no return value)
                __syncthreads();
                const uint64_t mw = (uint64_t)c * (kChunkWords / 32) + tid;
                if (tid < kChunkWords / 32 && s_mb[tid]) {
                    atomicOr(p.a.mask + mw, s_mb[tid]);
                    p.d.imask[mw] = s_mb[tid];  // (k_classify zeroed it; this CTA alone writes the chunk's words)
                }
            }
            __syncthreads();  // s_pre / s_mb are rewritten for the next chunk
        }
    }
    pdl_trigger();
    TL_REC(10, 0, tl0);
}

// ----------------------------------------------------------------------------
// 5. k_emit: the slot table (one CTA per kEmitChunks chunks, one thread per
//    output record: coalesced stores).  Record r of chunk c is the r-th set bit q
//    of its mask words; it comes from the window-hit region of the classify warp
//    that owned q if q is not in the I-resolved mask (rank among that warp's
//    window hits below q), else from its queue entry, where k_iresolve left it (rank among the
//    warp's queued words below q).  Regions are read in order: no word-indexed
//    staging.
// chunks per k_emit CTA: 2 (the grid of a large set fits one wave); 1 for a set of
// fewer than two chunks per SM (a single model's), whose CTAs then spread over
// more SMs with half the records each
template <int kEmitChunks>
__global__ void __launch_bounds__(kThreads) k_emit(P p) {
    __shared__ uint32_t s_m[kEmitChunks][64], s_i[kEmitChunks][64], s_q[kEmitChunks][64];
    __shared__ uint32_t s_pre[kEmitChunks][65], s_prm[kEmitChunks][65], s_prq[kEmitChunks][65];
    const unsigned long long tl0 = TL_NOW();
    unsigned long long tl_p = tl0;
    pdl_wait();
    if (MEDUSA_EARLY_TRIGGER) pdl_trigger();  // k_result waits for this grid's completion
    TL_PHASE(5, 60, tl_p);  // wait
    const MaterializeArgs& a = p.a;
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t c0 = blockIdx.x * kEmitChunks;
    const uint32_t nch = min((uint32_t)kEmitChunks, p.C - c0);
    const uint64_t n_mask = (a.n_words + 31) / 32;
    // the mask words (warps 0-3, one per lane), the chunks' counts and (in the same
    // load round) the first chunk's first slot: the sum of the slot counts of all
    // earlier chunks
    const uint32_t h_m = warp >> 1;
    const uint64_t mw_m = (uint64_t)(c0 + h_m) * (kChunkWords / 32) + (warp & 1) * 32 + lane;
    const bool in_m = warp < 2 * kEmitChunks && h_m < nch && mw_m < n_mask;
    const uint32_t mv_m = in_m ? __ldcg(a.mask + mw_m) : 0u, iv_m = in_m ? __ldcg(p.d.imask + mw_m) : 0u;
    const uint32_t qv_m = in_m ? __ldcg(p.d.qmask + mw_m) : 0u;
    uint32_t total[kEmitChunks];
#pragma unroll
    for (int h = 0; h < kEmitChunks; ++h) total[h] = (uint32_t)h < nch ? __ldcg(p.d.chunk_cnt + c0 + h) : 0u;
    uint64_t prefix = block_prefix(p.d.chunk_cnt, p.d.chunk_sup, c0);
    TL_PHASE(5, 61, tl_p);  // mask words, counts, chunk prefix
    if (warp < 2 * kEmitChunks) {  // popcount prefixes of each half of each chunk's 64 mask words
        const uint32_t h = h_m, half = warp & 1;
        const uint32_t mv = mv_m, iv = iv_m, qv = qv_m;
        const uint32_t x = half * 32 + lane;
        s_m[h][x] = mv;
        s_i[h][x] = iv;
        s_q[h][x] = qv;
        uint32_t c3[3] = {(uint32_t)__popc(mv), (uint32_t)__popc(mv & ~iv), (uint32_t)__popc(qv)};
        uint32_t* pre[3] = {s_pre[h], s_prm[h], s_prq[h]};
#pragma unroll
        for (int t = 0; t < 3; ++t) {
            uint32_t incl = c3[t];
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl += y;
            }
            pre[t][x] = incl - c3[t];
            if (half == 0 && lane == 31) pre[t][64] = incl;  // first-half total
        }
    }
    __syncthreads();
    if (tid >= 32 && tid < 64) {  // second halves after the first
#pragma unroll
        for (int h = 0; h < kEmitChunks; ++h) {
            s_pre[h][tid] += s_pre[h][64];
            s_prm[h][tid] += s_prm[h][64];
            s_prq[h][tid] += s_prq[h][64];
        }
    }
    __syncthreads();
    if (tid == 0) {
#pragma unroll
        for (int h = 0; h < kEmitChunks; ++h) {
            if ((uint32_t)h >= nch) break;
            const uint64_t pf = prefix + (h ? total[0] : 0u);
            a.chunk_base[c0 + h] = (uint32_t)pf;
            if (c0 + h + 1 == p.C) {
                a.chunk_base[c0 + h + 1] = (uint32_t)(pf + total[h]);
                p.d.ctl->n_slots = pf + total[h];
            }
        }
    }
    TL_PHASE(5, 62, tl_p);  // popcount prefixes, chunk_base
    // records: every load of the CTA's (up to kRecPerThread per chunk per thread)
    // issued before the first store -- the loads do not wait for each other
    constexpr int kRecPerThread = 2;
    auto source = [&](int h, uint32_t r) -> uint64_t {  // the record of the chunk's r-th slot
        uint32_t lo = 0;  // last mask word m with s_pre[m] <= r (s_pre[0] = 0): binary lifting, no branches
#pragma unroll
        for (uint32_t st = 32; st > 0; st >>= 1) lo += s_pre[h][lo + st] <= r ? st : 0u;
        MCHECK(lo < 64 && r >= s_pre[h][lo] && r - s_pre[h][lo] < (uint32_t)__popc(s_m[h][lo]));
        const uint32_t bit = nth_set_bit(s_m[h][lo], r - s_pre[h][lo]);  // the (r - s_pre[lo])-th set bit
        MCHECK(bit < 32 && ((s_m[h][lo] >> bit) & 1u));
        const uint32_t below = (1u << bit) - 1u;
        const uint32_t w = lo / 8;  // the classify warp that owned the word
        const uint64_t region = (uint64_t)((c0 + h) * kWarps + w) * p.d.cap_pw;
        if ((s_i[h][lo] >> bit) & 1u) {  // resolved by the I list: beside its queue entry
            const uint32_t k = s_prq[h][lo] - s_prq[h][w * 8] + __popc(s_q[h][lo] & below);
            return k < p.d.cap_pw ? __ldcg(&p.d.queue[region + k].x) : 0ull;
        }
        const uint32_t k = s_prm[h][lo] - s_prm[h][w * 8] + __popc(s_m[h][lo] & ~s_i[h][lo] & below);
        return k < p.d.cap_pw ? __ldcg(p.d.rec + region + k) : 0ull;
    };
    uint64_t val[kEmitChunks][kRecPerThread], dst[kEmitChunks][kRecPerThread];
#pragma unroll
    for (int h = 0; h < kEmitChunks; ++h) {
        const uint64_t pf = prefix + (h ? total[0] : 0u);
#pragma unroll
        for (int k = 0; k < kRecPerThread; ++k) {
            const uint32_t r = tid + k * kThreads;
            dst[h][k] = ~0ull;
            if (r < total[h] && pf + r < a.capacity) {
                dst[h][k] = pf + r;
                val[h][k] = source(h, r);
            }
        }
    }
#pragma unroll
    for (int h = 0; h < kEmitChunks; ++h)
#pragma unroll
        for (int k = 0; k < kRecPerThread; ++k)
            if (dst[h][k] != ~0ull) a.slot[dst[h][k]] = val[h][k];
    // the rest (chunks with more than kRecPerThread * kThreads records)
#pragma unroll
    for (int h = 0; h < kEmitChunks; ++h) {
        const uint64_t pf = prefix + (h ? total[0] : 0u);
        for (uint32_t r = tid + kRecPerThread * kThreads; r < total[h]; r += kThreads)
            if (pf + r < a.capacity) a.slot[pf + r] = source(h, r);
    }
    TL_PHASE(5, 63, tl_p);  // records
    if (!MEDUSA_EARLY_TRIGGER) pdl_trigger();
    TL_REC(5, 0, tl0);
}

// ----------------------------------------------------------------------------
// 6. k_result (async entry): the outcome as a medusa_mat_result
__global__ void k_result(P p, medusa_mat_result* r) {
    if (MEDUSA_EARLY_TRIGGER) pdl_trigger();
    pdl_wait();
    if (!MEDUSA_EARLY_TRIGGER) pdl_trigger();
    const Ctl& c = *p.d.ctl;
    int32_t st = MEDUSA_OK;
    if (c.status & ST_INVALID) st = MEDUSA_ERR_INVALID_ARG;
    else if (c.status & ST_TRACE) st = MEDUSA_ERR_TRACE;
    else if (c.status & ST_OVERFLOW) st = MEDUSA_ERR_RETRY;
    else if (c.n_slots > p.a.capacity) st = MEDUSA_ERR_CAPACITY;
    r->status = st;
    r->reserved = 0;
    r->n_slots = (st == MEDUSA_OK || st == MEDUSA_ERR_CAPACITY) ? c.n_slots : 0;
}

// ----------------------------------------------------------------------------
// host side: per-device scratch, launches

// level sizes of the mortal tree over n ordinals (cnt[0] = n; the top level has
// <= 32 nodes); node levels 1..top stored back to back
Tree tree_shape(uint64_t n) {
    Tree t{};
    t.cnt[0] = (uint32_t)n;
    uint32_t l = 0, o = 0;
    while (t.cnt[l] > 32 && l < (uint32_t)kMaxLevels) {
        t.cnt[l + 1] = (t.cnt[l] + 31) / 32;
        ++l;
        t.off[l] = o;
        o += t.cnt[l];
    }
    t.top = l;
    t.off[kMaxLevels] = o;  // (scratch sizing: total node count)
    return t;
}

struct Scratch {
    size_t cap_n = 0, cap_C = 0, cap_w = 0, cap_r = 0, cap_q = 0;
    void* zero_region = nullptr;
    size_t zero_bytes = 0;
    Dev d{};
    std::vector<void*> bufs;
    Ctl* h_ctl = nullptr;
    int sm_count = 0;
    cudaStream_t side = nullptr;  // the I-list sort + rank branch (highest priority; forked from the caller's stream)
    cudaStream_t low = nullptr;   // the trace-check branch (default priority; joined before the call ends)
    cudaEvent_t fork = nullptr, traced = nullptr, join = nullptr, ranked = nullptr, classified = nullptr,
                emitted = nullptr;
    // Buffers retired by a growth.  A CUDA graph that captured an earlier
    // medusa_materialize_async holds their addresses by value, so they stay
    // allocated (replaying such a graph stays memory-safe) until
    // medusa_scratch_release() or process exit.
    std::vector<void*> graveyard;
    size_t bytes = 0;  // live scratch bytes (zero region + buffers)
    std::mutex mu;  // one materialize at a time per device (the scratch is shared); devices run concurrently
};
std::mutex g_mu;  // guards g_scratch only
std::vector<Scratch*> g_scratch;

template <class T>
cudaError_t grow(Scratch& s, T*& p, size_t elems) {
    T* q = nullptr;
    cudaError_t e = cudaMalloc(&q, std::max<size_t>(elems, 1) * sizeof(T));
    if (e != cudaSuccess) return e;
    p = q;
    s.bufs.push_back(q);
    s.bytes += std::max<size_t>(elems, 1) * sizeof(T);
    return cudaSuccess;
}

// the current buffers -> the graveyard (not freed: see Scratch::graveyard)
void retire(Scratch& s) {
    for (void* p : s.bufs) s.graveyard.push_back(p);
    s.bufs.clear();
    if (s.zero_region) s.graveyard.push_back(s.zero_region);
    s.zero_region = nullptr;
    s.bytes = 0;
    s.cap_n = s.cap_C = s.cap_w = s.cap_r = s.cap_q = 0;
}

// grow geometrically (x1.5) past the previous capacity, so a sequence of growing
// calls retires a bounded amount of memory
size_t grown(size_t need, size_t old) { return need <= old ? old : std::max(need, old + old / 2); }

// Warp regions of 128 entries (half the warp's 256 words; the BASELINE sets:
// ~10% window hits and ~9% queued candidates, at most ~30% in any 256 words); a
// call whose warp needs more sets ST_OVERFLOW, and the synchronous entry reruns
// with regions of the whole warp (256, always enough).
constexpr size_t kRegion = 128;
cudaError_t ensure(Scratch& s, size_t n, size_t C, size_t W, size_t need_pw) {
    const size_t PC = need_pw > kRegion ? (size_t)(kChunkWords / kWarps) : kRegion;
    if (n <= s.cap_n && C <= s.cap_C && W <= s.cap_w && PC <= s.cap_r) return cudaSuccess;
    const size_t N = grown(std::max<size_t>(n, 1024), s.cap_n), CC = grown(std::max<size_t>(C, 64), s.cap_C);
    const size_t WW = grown(std::max<size_t>(W, 2048), s.cap_w);
    const size_t RR = std::max(PC, s.cap_r), QQ = CC * kWarps * RR;
    retire(s);
    const size_t NS = N / kIBlk + 1;
    const size_t NT = tree_shape(N).off[kMaxLevels] + 64;  // tree nodes (levels >= 1) for up to N ordinals
    cudaError_t e;
    // zero region: Ctl | chunk_sup [CC/256+1] (u64) | blk_min_ta_c blk_max_tf [NS] | chunk_cnt [CC] |
    //              tree nodes [NT] (uint2)
    const size_t GC = CC / 256 + 1;
    s.zero_bytes = (256 + GC * 8 + 2 * NS * 4 + CC * 4 + 64 + NT * 8 + 15) & ~(size_t)15;
    if ((e = cudaMalloc(&s.zero_region, s.zero_bytes)) != cudaSuccess) return e;
    s.bytes += s.zero_bytes;
    char* z = (char*)s.zero_region;
    s.d.ctl = (Ctl*)z;
    size_t o = 256;
    s.d.chunk_sup = (unsigned long long*)(z + o); o += GC * 8;
    s.d.blk_min_ta_c = (uint32_t*)(z + o); o += NS * 4;
    s.d.blk_max_tf = (uint32_t*)(z + o); o += NS * 4;
    s.d.chunk_cnt = (uint32_t*)(z + o); o += CC * 4;
    o = (o + 63) & ~(size_t)63;
    s.d.tree.node = (uint2*)(z + o);
    if ((e = grow(s, s.d.jf, CC)) || (e = grow(s, s.d.jl, CC)) || (e = grow(s, s.d.tree.leaf, N)) || (e = grow(s, s.d.tree.leaf_be, N)) ||
        (e = grow(s, s.d.sk0, N + kThreads)) || (e = grow(s, s.d.sv0, N + kThreads)) || (e = grow(s, s.d.sk, N)) ||
        (e = grow(s, s.d.sv, N)) || (e = grow(s, s.d.icnt, N / kThreads + 2)) ||
        (e = grow(s, s.d.tmax_k, N / kIsortTile + 2)) || (e = grow(s, s.d.tmax_v, N / kIsortTile + 2)) ||
        (e = grow(s, s.d.samp_k, N / kSampleStride + 64)) || (e = grow(s, s.d.samp_v, N / kSampleStride + 64)) ||
        (e = grow(s, s.d.i_base, N + 64)) || (e = grow(s, s.d.i_rest, N)) || (e = grow(s, s.d.i_tf, N)) ||
        (e = grow(s, s.d.fence, (size_t)kFenceCap)) ||
        (e = grow(s, s.d.rec, QQ)) || (e = grow(s, s.d.queue, QQ)) ||
        (e = grow(s, s.d.qcnt, CC * kWarps)) ||
        (e = grow(s, s.d.imask, WW / 32 + 1)) || (e = grow(s, s.d.qmask, WW / 32 + 1)))
        return e;
    // (the group scan reads whole 32-byte blocks, up to 7 bases past the list's end:
    // initialized once, their values are never used)
    if ((e = cudaMemset(s.d.i_base, 0, (N + 64) * sizeof(uint64_t)))) return e;
    s.d.cap_pw = (uint32_t)RR;
    s.cap_n = N; s.cap_C = CC; s.cap_w = WW; s.cap_r = RR; s.cap_q = QQ;
    return cudaSuccess;
}

}  // namespace

namespace {

// this device's scratch, returned with its lock held (*lk)
Scratch* device_scratch(cudaError_t* e, std::unique_lock<std::mutex>* lk) {
    int dev = 0;
    *e = cudaGetDevice(&dev);
    if (*e != cudaSuccess) return nullptr;
    Scratch* sp;
    {
        std::lock_guard<std::mutex> g(g_mu);
        if ((int)g_scratch.size() <= dev) g_scratch.resize(dev + 1, nullptr);
        if (!g_scratch[dev]) g_scratch[dev] = new Scratch();
        sp = g_scratch[dev];
    }
    *lk = std::unique_lock<std::mutex>(sp->mu);
    Scratch& s = *sp;
    if (!s.h_ctl) {
        if ((*e = cudaMallocHost(&s.h_ctl, sizeof(Ctl))) != cudaSuccess) return nullptr;
        cudaFuncSetAttribute(k_classify, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kClsSmem);
        cudaFuncSetAttribute(k_isort, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)(kIsortSmem + (kOrderedCtas + 1) * 4));
        int prio_lo = 0, prio_hi = 0;
        cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
        if ((*e = cudaStreamCreateWithPriority(&s.side, cudaStreamNonBlocking, prio_hi)) != cudaSuccess ||
            (*e = cudaStreamCreateWithPriority(&s.low, cudaStreamNonBlocking, prio_lo)) != cudaSuccess ||
            (*e = cudaEventCreateWithFlags(&s.fork, cudaEventDisableTiming)) != cudaSuccess ||
            (*e = cudaEventCreateWithFlags(&s.join, cudaEventDisableTiming)) != cudaSuccess ||
            (*e = cudaEventCreateWithFlags(&s.traced, cudaEventDisableTiming)) != cudaSuccess ||
            (*e = cudaEventCreateWithFlags(&s.ranked, cudaEventDisableTiming)) != cudaSuccess ||
            (*e = cudaEventCreateWithFlags(&s.classified, cudaEventDisableTiming)) != cudaSuccess ||
            (*e = cudaEventCreateWithFlags(&s.emitted, cudaEventDisableTiming)) != cudaSuccess)
            return nullptr;
        cudaDeviceGetAttribute(&s.sm_count, cudaDevAttrMultiProcessorCount, dev);
    }
    return &s;
}

cudaError_t launch_emit(const Scratch& s, uint32_t C, cudaStream_t st, const P& p) {
#ifndef MEDUSA_EMIT_SMALL
#define MEDUSA_EMIT_SMALL 1
#endif
    if (MEDUSA_EMIT_SMALL && C < 2u * (uint32_t)s.sm_count) return launch_pdl(k_emit<1>, C, kThreads, 0, st, p);
    return launch_pdl(k_emit<2>, (C + 1) / 2, kThreads, 0, st, p);
}

// the whole analysis on `stream` (no synchronization):
//   stream:            memset -> k_trace [traced] -> k_classify -> [ranked] k_iresolve -> k_emit [join]
//   side (high prio):             [traced] k_isort -> k_rank [ranked]
//   low (default):                [traced] k_check_mm ... [ranked] k_check_mi [join]
// The high-priority stream gets the sort / rank CTAs dispatched ahead of the
// classify CTAs and the queue resolution / emission ahead of the trace checks,
// which fill in around them and complete the call.
cudaError_t enqueue(Scratch& s, const MaterializeArgs& a, cudaStream_t stream, P* out) {
    const uint64_t n = a.n_alloc;
    const uint32_t C = (uint32_t)((a.n_words + kChunkWords - 1) / kChunkWords);
    const uint32_t nb = (uint32_t)((n + 31) / 32);
    const uint32_t node_ctas = (a.n_nodes + 1 + kThreads * kNodesPerThread - 1) / (kThreads * kNodesPerThread);
    const uint32_t alloc_ctas = (uint32_t)((n + kThreads - 1) / kThreads);
    const uint32_t sort_ctas = (uint32_t)((n + kIsortTile - 1) / kIsortTile);
    const uint32_t check_ctas = (nb + kWarps - 1) / kWarps;
    Dev d = s.d;
    const Tree shape = tree_shape(n);
    d.tree.top = shape.top;
    {  // the query's start level (q_start)
        int l = (int)shape.top;
        while (l > 0 && shape.cnt[l - 1] <= (uint32_t)kThreads) --l;
        d.tree.l0 = l;
    }
    for (int l = 0; l <= kMaxLevels; ++l) { d.tree.cnt[l] = shape.cnt[l]; d.tree.off[l] = shape.off[l]; }
    // ordinal-ordered I compaction pays when the set spans several address regions
    // (several models: most rank tiles then hold another model's keys); a single
    // model's set (<= 128 k_trace CTAs, ~4 tiles) skips the gather it costs k_isort
#ifndef MEDUSA_ORDERED_MIN_CTAS
#define MEDUSA_ORDERED_MIN_CTAS 128
#endif
    const uint32_t ordered = (alloc_ctas > MEDUSA_ORDERED_MIN_CTAS && alloc_ctas <= kOrderedCtas) ? 1u : 0u;
    P p{a, d, C, nb, node_ctas, alloc_ctas, ordered};
    *out = p;
    cudaError_t e;
    // branches (serialized on the caller's stream while per-launch timing is on)
    const bool serial = timing_enabled();
    cudaStream_t side = serial ? stream : s.side, low = serial ? stream : s.low;
#ifndef MEDUSA_ZERO_KERNEL
#define MEDUSA_ZERO_KERNEL 1
#endif
    if (C == 0 && (e = cudaMemsetAsync(a.chunk_base, 0, sizeof(uint32_t), stream)) != cudaSuccess) return e;
    if (MEDUSA_ZERO_KERNEL) {
        const size_t n16 = s.zero_bytes / 16;  // (zero_bytes: a multiple of 16)
        {
            TimedLaunch tl("mat_zero", stream);
            if ((e = launch_pdl(k_zero, (unsigned)std::min<size_t>((n16 + kThreads - 1) / kThreads, (size_t)s.sm_count * 2),
                                kThreads, 0, stream, reinterpret_cast<uint4*>(s.zero_region), n16)))
                return e;
        }
        TimedLaunch tl("mat_trace", stream);
        if ((e = launch_pdl(k_trace, node_ctas + alloc_ctas, kThreads, 0, stream, p))) return e;
    } else {
        if ((e = cudaMemsetAsync(s.zero_region, 0, s.zero_bytes, stream)) != cudaSuccess) return e;
        TimedLaunch tl("mat_trace", stream);
        k_trace<<<node_ctas + alloc_ctas, kThreads, 0, stream>>>(p);
    }
    if (n) {
        if ((e = cudaEventRecord(s.traced, stream)) || (e = cudaStreamWaitEvent(side, s.traced, 0))) return e;
        {
            TimedLaunch tl("mat_isort", side);
            k_isort<<<sort_ctas, kIsortThreads, kIsortSmem + (ordered ? (alloc_ctas + 1) * 4 : 0), side>>>(p);
        }
        if (n > (uint64_t)kIsortTile) {  // (with one tile k_isort writes the I list itself)
            TimedLaunch tl("mat_rank", side);
            // one CTA per 32 I keys (the list's size is known on the device only: bound
            // by the allocation count; surplus CTAs exit at once)
            if ((e = launch_pdl(k_rank, (unsigned)std::min<uint64_t>((n + 31) / 32, (uint64_t)s.sm_count * 8), kThreads,
                                0, side, p)))
                return e;
        }
        if ((e = cudaEventRecord(s.ranked, side))) return e;
    }
    if (C) {
        TimedLaunch tl("mat_classify", stream);
        if ((e = launch_pdl(k_classify, C, kThreads, kClsSmem, stream, p))) return e;
    }
#ifndef MEDUSA_MAIN_TAIL
#define MEDUSA_MAIN_TAIL 1  // (0: on the side stream, joined: ALL10 +1.5 us, C5 +1.2 us)
#endif
    if (n) {
        if (MEDUSA_MAIN_TAIL) {
            // the caller's stream after the classify and the rank: queue resolution and
            // emission, so k_result and a following restore are their programmatic successors
            if ((e = cudaStreamWaitEvent(stream, s.ranked, 0))) return e;
            if (C) {
                {
                    TimedLaunch tl("mat_iresolve", stream);
#ifndef MEDUSA_IRES_PER_SM
#define MEDUSA_IRES_PER_SM 6
#endif
                    if ((e = launch_pdl(k_iresolve, std::min<unsigned>(C, (unsigned)s.sm_count * MEDUSA_IRES_PER_SM),
                                        kThreads, 0, stream, p)))
                        return e;
                }
                TimedLaunch tl("mat_emit", stream);
                if ((e = launch_emit(s, C, stream, p))) return e;
            }
        } else {
            if ((e = cudaEventRecord(s.classified, stream))) return e;
            // high priority after the classify: queue resolution and emission (the
            // rank is already on this stream)
            if ((e = cudaStreamWaitEvent(side, s.classified, 0))) return e;
            if (C) {
                {
                    TimedLaunch tl("mat_iresolve", side);
                    k_iresolve<<<std::min<unsigned>(C, (unsigned)s.sm_count * 6), kThreads, 0, side>>>(p);  // one wave (6 per SM)
                }
                TimedLaunch tl("mat_emit", side);
                if ((e = launch_emit(s, C, side, p))) return e;
            }
            if ((e = cudaEventRecord(s.emitted, side))) return e;
        }
        // default priority: the trace checks fill in around them (M-M needs the
        // mortal tree only, M-I and I-I the sorted I list)
        if ((e = cudaStreamWaitEvent(low, s.traced, 0))) return e;
#ifndef MEDUSA_DIAG_NO_CHECKS  // (diagnostic builds only: the step without the R-Q7 checks)
        {
            TimedLaunch tl("mat_check_mm", low);
            k_check_mm<<<check_ctas, kThreads, 0, low>>>(p);
        }
#endif
        if ((e = cudaStreamWaitEvent(low, s.ranked, 0))) return e;
#ifndef MEDUSA_DIAG_NO_CHECKS
        {
            TimedLaunch tl("mat_check_mi", low);
            k_check_mi<<<check_ctas, kThreads, 0, low>>>(p);
        }
#endif
        if ((e = cudaEventRecord(s.join, low))) return e;
        if (!MEDUSA_MAIN_TAIL && (e = cudaStreamWaitEvent(stream, s.emitted, 0))) return e;
        if ((e = cudaStreamWaitEvent(stream, s.join, 0))) return e;
    } else if (C) {
        TimedLaunch tl("mat_emit", stream);
        if ((e = launch_emit(s, C, stream, p))) return e;
    }
    return cudaGetLastError();
}

}  // namespace

medusa_status run_materialize(const MaterializeArgs& a, uint64_t* n_slots, cudaStream_t stream,
                              cudaError_t* cuda_err) {
    *n_slots = 0;
    cudaError_t e;
    std::unique_lock<std::mutex> lk;  // this device's scratch, for the whole call (other devices run concurrently)
    Scratch* sp = device_scratch(&e, &lk);
    if (!sp) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    Scratch& s = *sp;
    const uint32_t C = (uint32_t)((a.n_words + kChunkWords - 1) / kChunkWords);
    size_t need_pw = 0;
    for (int attempt = 0; attempt < 2; ++attempt) {
        P p;
        if ((e = ensure(s, a.n_alloc, C, a.n_words, need_pw)) != cudaSuccess ||
            (e = enqueue(s, a, stream, &p)) != cudaSuccess ||
            (e = cudaMemcpyAsync(s.h_ctl, s.d.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, stream)) != cudaSuccess ||
            (e = cudaStreamSynchronize(stream)) != cudaSuccess) {
            *cuda_err = e;
            return MEDUSA_ERR_CUDA;
        }
        const Ctl h = *s.h_ctl;
        if (h.status & ST_INVALID) return MEDUSA_ERR_INVALID_ARG;
        if (h.status & ST_TRACE) return MEDUSA_ERR_TRACE;
        if (h.status & ST_OVERFLOW) {  // a warp's record / queue region too small: whole-warp regions, rerun
            need_pw = std::max<size_t>(need_pw, h.need_pw);
            continue;
        }
        *n_slots = h.n_slots;
        return h.n_slots > a.capacity ? MEDUSA_ERR_CAPACITY : MEDUSA_OK;
    }
    *cuda_err = cudaErrorUnknown;  // (the exact sizes cannot overflow)
    return MEDUSA_ERR_CUDA;
}

medusa_status run_materialize_async(const MaterializeArgs& a, medusa_mat_result* d_result, cudaStream_t stream,
                                    cudaError_t* cuda_err) {
    cudaError_t e;
    std::unique_lock<std::mutex> lk;  // held while enqueueing only
    Scratch* sp = device_scratch(&e, &lk);
    if (!sp) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    Scratch& s = *sp;
    const uint32_t C = (uint32_t)((a.n_words + kChunkWords - 1) / kChunkWords);
    // never (re)allocates while the caller may be capturing a graph, unless it must grow
    if ((e = ensure(s, a.n_alloc, C, a.n_words, 0)) != cudaSuccess) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    P p;
    if ((e = enqueue(s, a, stream, &p)) != cudaSuccess) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    if ((e = launch_pdl(k_result, 1, 1, 0, stream, p, d_result))) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    if ((e = cudaGetLastError()) != cudaSuccess) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    return MEDUSA_OK;
}

uint64_t scratch_bytes() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return 0;
    std::lock_guard<std::mutex> g(g_mu);
    if ((int)g_scratch.size() <= dev || !g_scratch[dev]) return 0;
    return g_scratch[dev]->bytes;
}

cudaError_t release_scratch() {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    Scratch* sp = nullptr;
    {
        std::lock_guard<std::mutex> g(g_mu);
        if ((int)g_scratch.size() > dev) sp = g_scratch[dev];
    }
    if (!sp) return cudaSuccess;
    std::lock_guard<std::mutex> lk(sp->mu);
    if ((e = cudaDeviceSynchronize()) != cudaSuccess) return e;
    retire(*sp);
    for (void* p : sp->graveyard) cudaFree(p);
    sp->graveyard.clear();
    return cudaGetLastError();
}

}  // namespace medusa

#ifdef MEDUSA_TIMELINE
extern "C" int medusa_tl_attach_mat(void* buf, unsigned cap) {
    unsigned zero = 0;
    medusa::TlRec* b = static_cast<medusa::TlRec*>(buf);
    if (cudaMemcpyToSymbol(medusa::g_tl, &b, sizeof(b)) != cudaSuccess) return -1;
    if (cudaMemcpyToSymbol(medusa::g_tl_cap, &cap, sizeof(cap)) != cudaSuccess) return -1;
    return cudaMemcpyToSymbol(medusa::g_tl_n, &zero, sizeof(zero)) == cudaSuccess ? 0 : -1;
}
extern "C" unsigned medusa_tl_count_mat() {
    unsigned n = 0;
    cudaMemcpyFromSymbol(&n, medusa::g_tl_n, sizeof(n));
    return n;
}
#endif
