// MATERIALIZE: indirect-index-pointer analysis (§4.1) on
// sm_100a.  For every 8-byte word w of node j (launched at t_j), find the
// allocation i live at the launch (t_alloc_i < t_j < t_free_i) whose range
// [base_i, base_i + size_i) holds w ("identical or within the range");
// emit the indirect index pointer table in word order.
//
// Structure of a well-formed trace that the GPU design exploits:
//  * I = allocations live at the LAST launch T_last.  All of them are live at
//    the same instant, so they are pairwise address-disjoint: one global list
//    sorted by base answers "which I-allocation holds w" with one binary search;
//    it is live at t <= T_last iff t_alloc < t.  (weights, KV cache, static
//    inputs, permanent buffers: ~27k entries for the ten-model set.)
//  * M = every other allocation ("mortal": capture temporaries, warm-up and
//    profiling scratch).  Their lifetimes are short, so each is registered in
//    the word chunks whose launch-time span its lifetime touches; a chunk's
//    mortal window (~60-150 entries) is sorted by base in shared memory and
//    searched with a prefix-max-of-end backward walk plus the time check.
//  * Well-formedness (no two simultaneously-live allocations overlap) is checked
//    exactly: I-I by adjacency of the sorted list, M-I by an address-run walk
//    over the sorted I list, M-M inside blocks of 64 allocation ordinals
//    against the mortals registered as live there.
// Pipeline (all on `stream`; one host synchronization at the end):
//   k_nodes_chunks  CSR / launch-order checks, per-chunk launch-time span
//   k_allocs        trace checks, I/M split, registration counts, prefilter
//   k_scan          registration offsets (single CTA)
//   k_scatter       registration lists
//   k_sort_tile + k_merge (x log)   I sorted by (base, index)
//   k_build_i       I arrays, I-I check, fences
//   k_check         M-M and M-I overlap checks
//   k_classify      classify every word + ballot/popc emission with a decoupled
//                   look-back over chunks (persistent CTAs, ticketed chunks)
#include <algorithm>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace medusa {
namespace {

constexpr uint32_t ST_INVALID = 1, ST_TRACE = 2, ST_OVERFLOW = 4;
constexpr int kAblk = 64;          // allocation ordinals per overlap-check block
constexpr int kChkCap = 1024;      // registered mortals staged per check batch
constexpr int kSortTile = 2048;
constexpr int kFenceCap = 2048;    // I-list fences held in shared memory
constexpr int kWinCap = 512;       // mortal-window entries per batch (power of two)
constexpr int kClsThreads = 256;
constexpr int kWordsPerThread = MEDUSA_CHUNK_WORDS / kClsThreads;  // 8
constexpr int kWarps = kClsThreads / 32;
constexpr unsigned long long LB_AGG = 1ull << 62, LB_PRE = 2ull << 62, LB_VAL = (1ull << 62) - 1;

struct Ctl {
    unsigned int status;
    unsigned int nI;
    unsigned int ticket;
    unsigned int pad;
    unsigned long long gmin_c;  // ~(least base) via atomicMax
    unsigned long long gmax;    // greatest end
    unsigned long long need_c, need_b;
    unsigned long long n_slots;
};

struct IRest {
    uint64_t end;
    uint32_t t_alloc;
    uint32_t id;
};

struct Dev {  // scratch of one call (device pointers)
    Ctl* ctl;
    uint32_t *tmin, *tmax, *jf, *jl;             // [C]
    uint4* rng;                                  // [n]: c_lo, c_hi, b_lo, b_hi
    uint32_t *cnt_c, *fill_c, *off_c;            // [C+1]
    uint32_t *cnt_b, *fill_b, *off_b;            // [nb+1]
    uint32_t *list_c, *list_b;
    uint64_t cap_c, cap_b;
    uint64_t *sk0, *sk1;                         // [n] sort keys
    uint32_t *sv0, *sv1;                         // [n] sort values
    uint64_t* i_base;                            // [n]
    IRest* i_rest;                               // [n]
    uint64_t* fence;                             // [kFenceCap]
    unsigned long long* lookback;                // [C]
};

struct P {  // kernel parameters
    MaterializeArgs a;
    Dev d;
    uint32_t C, nb;
};

__device__ __forceinline__ void flag(Ctl* c, unsigned int bit) { atomicOr(&c->status, bit); }

// largest j in [0, N-1] with node_off[j] <= g (N >= 1)
__device__ __forceinline__ uint32_t node_of(const uint64_t* off, uint32_t N, uint64_t g) {
    uint32_t lo = 0, hi = N;  // count of node_off[1..N] <= g
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (off[mid + 1] <= g) lo = mid + 1; else hi = mid;
    }
    return lo < N ? lo : N - 1;
}

__device__ __forceinline__ bool kv_less(uint64_t ka, uint32_t va, uint64_t kb, uint32_t vb) {
    return ka < kb || (ka == kb && va < vb);
}

__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// ----------------------------------------------------------------------------
// 1. nodes and chunks
__global__ void k_nodes_chunks(P p) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const MaterializeArgs& a = p.a;
    const uint32_t N = a.n_nodes;
    if (i <= N) {
        if (i == 0 && a.node_off[0] != 0) flag(p.d.ctl, ST_INVALID);
        if (i == N && a.node_off[N] != a.n_words) flag(p.d.ctl, ST_INVALID);
        if (i < N && a.node_off[i + 1] < a.node_off[i]) flag(p.d.ctl, ST_INVALID);
        if (i + 1 < N && !(a.node_t[i] < a.node_t[i + 1])) flag(p.d.ctl, ST_INVALID);
    }
    if (i < p.C && N > 0) {
        const uint64_t cs = i * kChunkWords;
        const uint64_t ce = min(cs + kChunkWords, a.n_words) - 1;
        const uint32_t jf = node_of(a.node_off, N, cs), jl = node_of(a.node_off, N, ce);
        p.d.jf[i] = jf;
        p.d.jl[i] = jl;
        p.d.tmin[i] = a.node_t[jf];
        p.d.tmax[i] = a.node_t[jl];
    }
}

// ----------------------------------------------------------------------------
// 2. allocations: checks, I/M split, registration ranges and counts
__global__ void k_allocs(P p) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    const MaterializeArgs& a = p.a;
    if (i >= a.n_alloc) return;
    const medusa_alloc x = a.alloc[i];
    if (x.size > (1ull << MEDUSA_OFF_BITS) || x.base + x.size < x.base) flag(p.d.ctl, ST_INVALID);
    if (!(x.t_alloc < x.t_free)) flag(p.d.ctl, ST_TRACE);
    if (i + 1 < a.n_alloc && !(x.t_alloc < a.alloc[i + 1].t_alloc)) flag(p.d.ctl, ST_TRACE);
    uint4 r = make_uint4(1, 0, 1, 0);  // empty ranges
    if (x.size != 0) {
        atomicMax(&p.d.ctl->gmin_c, ~(unsigned long long)x.base);
        atomicMax(&p.d.ctl->gmax, (unsigned long long)(x.base + x.size));
        const uint32_t N = a.n_nodes;
        const uint32_t t_last = N ? a.node_t[N - 1] : 0;
        if (N && x.t_alloc < t_last && t_last < x.t_free) {
            const unsigned int pos = atomicAdd(&p.d.ctl->nI, 1u);
            p.d.sk0[pos] = x.base;
            p.d.sv0[pos] = i;
        } else {
            if (p.C && N) {
                uint32_t lo = 0, hi = p.C;  // first chunk whose last launch is after t_alloc
                while (lo < hi) { uint32_t m = (lo + hi) >> 1; if (p.d.tmax[m] > x.t_alloc) hi = m; else lo = m + 1; }
                const uint32_t c_lo = lo;
                lo = 0; hi = p.C;  // chunks whose first launch is before t_free
                while (lo < hi) { uint32_t m = (lo + hi) >> 1; if (p.d.tmin[m] < x.t_free) lo = m + 1; else hi = m; }
                if (c_lo < lo) {
                    r.x = c_lo; r.y = lo - 1;
                    for (uint32_t c = r.x; c <= r.y; ++c) atomicAdd(&p.d.cnt_c[c], 1u);
                }
            }
            // ordinals allocated while i is live: (i, u) with u = #{k : t_alloc_k < t_free_i}
            uint32_t lo = i + 1, hi = a.n_alloc;
            while (lo < hi) { uint32_t m = (lo + hi) >> 1; if (a.alloc[m].t_alloc < x.t_free) lo = m + 1; else hi = m; }
            if (i + 1 < lo) {
                r.z = (i + 1) / kAblk; r.w = (lo - 1) / kAblk;
                for (uint32_t b = r.z; b <= r.w; ++b) atomicAdd(&p.d.cnt_b[b], 1u);
            }
        }
    }
    p.d.rng[i] = r;
}

// ----------------------------------------------------------------------------
// 3. exclusive scans of the registration counts (one CTA)
__device__ void block_exclusive_scan(const uint32_t* cnt, uint32_t* off, uint32_t n, unsigned long long* total) {
    __shared__ unsigned long long s_part[1024];
    const uint32_t T = blockDim.x, tid = threadIdx.x;
    const uint32_t per = (n + T - 1) / T;
    const uint32_t b = tid * per, e = min(b + per, n);
    unsigned long long s = 0;
    for (uint32_t k = b; k < e; ++k) s += cnt[k];
    s_part[tid] = s;
    __syncthreads();
    for (uint32_t d = 1; d < T; d <<= 1) {
        unsigned long long v = tid >= d ? s_part[tid - d] : 0;
        __syncthreads();
        s_part[tid] += v;
        __syncthreads();
    }
    unsigned long long run = s_part[tid] - s;
    for (uint32_t k = b; k < e; ++k) { off[k] = (uint32_t)min(run, 0xFFFFFFFFull); run += cnt[k]; }
    if (tid == T - 1) { *total = s_part[T - 1]; off[n] = (uint32_t)min(s_part[T - 1], 0xFFFFFFFFull); }
    __syncthreads();
}

__global__ void __launch_bounds__(1024) k_scan(P p) {
    block_exclusive_scan(p.d.cnt_c, p.d.off_c, p.C, &p.d.ctl->need_c);
    block_exclusive_scan(p.d.cnt_b, p.d.off_b, p.nb, &p.d.ctl->need_b);
    if (threadIdx.x == 0 && (p.d.ctl->need_c > p.d.cap_c || p.d.ctl->need_b > p.d.cap_b))
        flag(p.d.ctl, ST_OVERFLOW);
}

// 4. registration lists
__global__ void k_scatter(P p) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= p.a.n_alloc) return;
    const uint4 r = p.d.rng[i];
    for (uint32_t c = r.x; c <= r.y; ++c) {
        const uint64_t pos = (uint64_t)p.d.off_c[c] + atomicAdd(&p.d.fill_c[c], 1u);
        if (pos < p.d.cap_c) p.d.list_c[pos] = i;
    }
    for (uint32_t b = r.z; b <= r.w; ++b) {
        const uint64_t pos = (uint64_t)p.d.off_b[b] + atomicAdd(&p.d.fill_b[b], 1u);
        if (pos < p.d.cap_b) p.d.list_b[pos] = i;
    }
}

// ----------------------------------------------------------------------------
// 5. sort I by (base, index): bitonic tiles of 2048, then merge-path passes
__global__ void __launch_bounds__(1024) k_sort_tile(const Ctl* ctl, const uint64_t* kin, const uint32_t* vin,
                                                    uint64_t* kout, uint32_t* vout) {
    __shared__ uint64_t sk[kSortTile];
    __shared__ uint32_t sv[kSortTile];
    const uint32_t n = ctl->nI;
    const uint32_t t0 = blockIdx.x * kSortTile;
    if (t0 >= n) return;
    for (uint32_t q = threadIdx.x; q < kSortTile; q += blockDim.x) {
        const bool in = t0 + q < n;
        sk[q] = in ? kin[t0 + q] : ~0ull;
        sv[q] = in ? vin[t0 + q] : 0xFFFFFFFFu;
    }
    __syncthreads();
    for (uint32_t size = 2; size <= kSortTile; size <<= 1) {
        for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
            for (uint32_t q = threadIdx.x; q < kSortTile / 2; q += blockDim.x) {
                const uint32_t lo = 2 * q - (q & (stride - 1));
                const uint32_t hi = lo + stride;
                const bool up = (lo & size) == 0;
                const uint64_t ka = sk[lo], kb = sk[hi];
                const uint32_t va = sv[lo], vb = sv[hi];
                if (kv_less(kb, vb, ka, va) == up) { sk[lo] = kb; sk[hi] = ka; sv[lo] = vb; sv[hi] = va; }
            }
            __syncthreads();
        }
    }
    for (uint32_t q = threadIdx.x; q < kSortTile && t0 + q < n; q += blockDim.x) {
        kout[t0 + q] = sk[q];
        vout[t0 + q] = sv[q];
    }
}

__global__ void __launch_bounds__(256) k_merge(const Ctl* ctl, const uint64_t* kin, const uint32_t* vin,
                                               uint64_t* kout, uint32_t* vout, uint32_t width) {
    __shared__ uint64_t sk[kSortTile];
    __shared__ uint32_t sv[kSortTile];
    __shared__ uint32_t s_i0, s_i1;
    const uint32_t n = ctl->nI;
    const uint32_t o0 = blockIdx.x * kSortTile;
    if (o0 >= n) return;
    const uint32_t ps = o0 / (2 * width) * (2 * width);
    const uint32_t a0 = ps, a1 = min(ps + width, n), b0 = a1, b1 = min(ps + 2 * width, n);
    const uint32_t o1 = min(o0 + kSortTile, n);
    if (a1 >= b1) {  // lone run: copy
        for (uint32_t q = o0 + threadIdx.x; q < o1; q += blockDim.x) { kout[q] = kin[q]; vout[q] = vin[q]; }
        return;
    }
    const uint32_t la = a1 - a0, lb = b1 - b0;
    if (threadIdx.x < 2) {
        const uint32_t d = (threadIdx.x == 0 ? o0 : o1) - ps;
        uint32_t lo = d > lb ? d - lb : 0, hi = min(d, la);
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (kv_less(kin[b0 + d - 1 - mid], vin[b0 + d - 1 - mid], kin[a0 + mid], vin[a0 + mid])) hi = mid;
            else lo = mid + 1;
        }
        if (threadIdx.x == 0) s_i0 = lo; else s_i1 = lo;
    }
    __syncthreads();
    const uint32_t i0 = s_i0, i1 = s_i1;
    const uint32_t j0 = (o0 - ps) - i0, j1 = (o1 - ps) - i1;
    const uint32_t na = i1 - i0, nbb = j1 - j0;
    for (uint32_t q = threadIdx.x; q < na + nbb; q += blockDim.x) {
        const uint32_t src = q < na ? a0 + i0 + q : b0 + j0 + (q - na);
        sk[q] = kin[src];
        sv[q] = vin[src];
    }
    __syncthreads();
    // sa = sk[0..na), sb = sk[na..na+nbb); each thread merges 8 outputs
    const uint32_t per = kSortTile / 256;
    const uint32_t d = threadIdx.x * per;
    if (d < na + nbb) {
        uint32_t lo = d > nbb ? d - nbb : 0, hi = min(d, na);
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (kv_less(sk[na + d - 1 - mid], sv[na + d - 1 - mid], sk[mid], sv[mid])) hi = mid;
            else lo = mid + 1;
        }
        uint32_t ia = lo, ib = d - lo;
        for (uint32_t q = 0; q < per && d + q < na + nbb; ++q) {
            bool takeA = ib >= nbb || (ia < na && kv_less(sk[ia], sv[ia], sk[na + ib], sv[na + ib]));
            const uint32_t s = takeA ? ia++ : na + ib++;
            kout[o0 + d + q] = sk[s];
            vout[o0 + d + q] = sv[s];
        }
    }
}

// 6. I arrays, I-I adjacency check, shared-memory fences
__global__ void k_build_i(P p, const uint64_t* sk, const uint32_t* sv) {
    const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
    const uint32_t nI = p.d.ctl->nI;
    if (k >= nI) return;
    const uint32_t id = sv[k];
    const medusa_alloc x = p.a.alloc[id];
    p.d.i_base[k] = x.base;
    p.d.i_rest[k] = IRest{x.base + x.size, x.t_alloc, id};
    if (k + 1 < nI && x.base + x.size > sk[k + 1]) flag(p.d.ctl, ST_TRACE);
    const uint32_t stride = (nI + kFenceCap - 1) / kFenceCap;
    if (k % stride == 0) p.d.fence[k / stride] = x.base;
}

// ----------------------------------------------------------------------------
// 7. overlap checks for mortal allocations
__global__ void __launch_bounds__(kAblk) k_check(P p) {
    __shared__ uint64_t s_base[kChkCap], s_end[kChkCap];
    __shared__ uint32_t s_tf[kChkCap], s_idx[kChkCap];
    const MaterializeArgs& a = p.a;
    const uint32_t b = blockIdx.x;
    const uint32_t j = b * kAblk + threadIdx.x;
    bool mine = false;
    medusa_alloc x{};
    const uint32_t N = a.n_nodes;
    const uint32_t t_last = N ? a.node_t[N - 1] : 0;
    if (j < a.n_alloc) {
        x = a.alloc[j];
        mine = x.size != 0 && !(N && x.t_alloc < t_last && t_last < x.t_free);
    }
    bool bad = false;
    // M-M: registered mortals live at some allocation of this block
    const uint64_t r0 = p.d.off_b[b];
    const uint64_t r1 = min((uint64_t)p.d.off_b[b + 1], p.d.cap_b);
    for (uint64_t bs = r0; bs < r1; bs += kChkCap) {
        const uint32_t m = (uint32_t)min((uint64_t)kChkCap, r1 - bs);
        __syncthreads();
        for (uint32_t q = threadIdx.x; q < m; q += blockDim.x) {
            const uint32_t i = p.d.list_b[bs + q];
            const medusa_alloc y = a.alloc[i];
            s_base[q] = y.base;
            s_end[q] = y.base + y.size;
            s_tf[q] = y.t_free;
            s_idx[q] = i;
        }
        __syncthreads();
        if (mine && !bad) {
            const uint64_t xe = x.base + x.size;
            for (uint32_t q = 0; q < m; ++q) {
                if (s_idx[q] < j && s_tf[q] > x.t_alloc && s_base[q] < xe && x.base < s_end[q]) { bad = true; break; }
            }
        }
    }
    // M-I: the I entries whose ranges meet [base, end) form one run of the sorted list
    if (mine && !bad) {
        const uint32_t nI = p.d.ctl->nI;
        const uint64_t xe = x.base + x.size;
        uint32_t lo = 0, hi = nI;  // count of I bases < xe
        while (lo < hi) { uint32_t m = (lo + hi) >> 1; if (p.d.i_base[m] < xe) lo = m + 1; else hi = m; }
        for (int64_t k = (int64_t)lo - 1; k >= 0; --k) {
            const IRest e = p.d.i_rest[k];
            if (e.end <= x.base) break;
            const uint32_t tf_e = a.alloc[e.id].t_free;
            if (max(e.t_alloc, x.t_alloc) < min(tf_e, x.t_free)) { bad = true; break; }
        }
    }
    if (bad) flag(p.d.ctl, ST_TRACE);
}

// ----------------------------------------------------------------------------
// 8. classify + emit
struct ClsShared {
    uint64_t fence[kFenceCap];
    uint32_t tw[MEDUSA_CHUNK_WORDS];
    uint64_t key[kWinCap];
    uint64_t end[kWinCap];
    uint64_t pmax[kWinCap];
    uint32_t ta[kWinCap], tf[kWinCap], id[kWinCap];
    uint16_t val[kWinCap];
    uint32_t cnt[kWordsPerThread][kWarps];
    uint32_t thr_max[kClsThreads];
    uint32_t chunk;
    unsigned long long prefix;
};

__global__ void __launch_bounds__(kClsThreads) k_classify(P p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    ClsShared& S = *reinterpret_cast<ClsShared*>(smem_raw);
    const MaterializeArgs& a = p.a;
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    Ctl* ctl = p.d.ctl;
    const uint32_t nI = ctl->nI;
    const uint32_t stride = nI ? (nI + kFenceCap - 1) / kFenceCap : 1;
    const uint32_t nf = (nI + stride - 1) / stride;
    for (uint32_t f = tid; f < nf; f += kClsThreads) S.fence[f] = p.d.fence[f];
    const uint64_t gmin = ~ctl->gmin_c, gmax = ctl->gmax;
    const uint32_t N = a.n_nodes;
    const uint64_t n_mask = (a.n_words + 31) / 32;

    for (;;) {
        __syncthreads();
        if (tid == 0) S.chunk = atomicAdd(&ctl->ticket, 1u);
        __syncthreads();
        const uint32_t c = S.chunk;
        if (c >= p.C) break;
        const uint64_t cs = (uint64_t)c * kChunkWords;
        const uint32_t n = (uint32_t)min((uint64_t)kChunkWords, a.n_words - cs);
        // words first: their latency overlaps everything below
        uint64_t w[kWordsPerThread];
#pragma unroll
        for (int k = 0; k < kWordsPerThread; ++k) {
            const uint32_t q = k * kClsThreads + tid;
            w[k] = q < n ? ld_stream(a.words + cs + q) : 0;
        }
        // launch position of every word: node starts carry t_j, then a max-scan
        for (uint32_t q = tid; q < kChunkWords; q += kClsThreads) S.tw[q] = 0;
        __syncthreads();
        if (N) {
            const uint32_t jf = p.d.jf[c], jl = p.d.jl[c];
            if (tid == 0) atomicMax(&S.tw[0], a.node_t[jf]);
            for (uint32_t j = jf + 1 + tid; j <= jl; j += kClsThreads) {
                const uint64_t q = a.node_off[j] - cs;
                if (q < n) atomicMax(&S.tw[q], a.node_t[j]);
            }
        }
        __syncthreads();
        {
            uint32_t loc[kWordsPerThread];
            uint32_t run = 0;
#pragma unroll
            for (int k = 0; k < kWordsPerThread; ++k) { run = max(run, S.tw[tid * kWordsPerThread + k]); loc[k] = run; }
            uint32_t incl = run;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl = max(incl, y);
            }
            S.thr_max[tid] = incl;  // inclusive within the warp
            __syncthreads();
            const uint32_t up = __shfl_up_sync(0xffffffffu, incl, 1);
            uint32_t before = lane ? up : 0;
            for (uint32_t ww = 0; ww < warp; ++ww) before = max(before, S.thr_max[ww * 32 + 31]);
            __syncthreads();
#pragma unroll
            for (int k = 0; k < kWordsPerThread; ++k) S.tw[tid * kWordsPerThread + k] = max(before, loc[k]);
        }
        __syncthreads();
        uint32_t t[kWordsPerThread];
        bool cand[kWordsPerThread], hit[kWordsPerThread];
        uint32_t hid[kWordsPerThread];
        uint64_t hoff[kWordsPerThread];
#pragma unroll
        for (int k = 0; k < kWordsPerThread; ++k) {
            const uint32_t q = k * kClsThreads + tid;
            t[k] = S.tw[q];
            cand[k] = q < n && w[k] >= gmin && w[k] < gmax;
            hit[k] = false;
            hid[k] = 0;
            hoff[k] = 0;
        }
        // mortal window(s): sorted by base, prefix max of end, backward walk
        const uint64_t r0 = p.d.off_c[c];
        const uint64_t r1 = min((uint64_t)p.d.off_c[c + 1], p.d.cap_c);
        for (uint64_t bs = r0; bs < r1; bs += kWinCap) {
            const uint32_t m = (uint32_t)min((uint64_t)kWinCap, r1 - bs);
            uint32_t mp = 32;
            while (mp < m) mp <<= 1;
            __syncthreads();
            for (uint32_t q = tid; q < mp; q += kClsThreads) {
                if (q < m) {
                    const uint32_t aid = p.d.list_c[bs + q];
                    const medusa_alloc x = a.alloc[aid];
                    S.key[q] = x.base;
                    S.end[q] = x.base + x.size;
                    S.ta[q] = x.t_alloc;
                    S.tf[q] = x.t_free;
                    S.id[q] = aid;
                } else {
                    S.key[q] = ~0ull;
                }
                S.val[q] = (uint16_t)q;
            }
            __syncthreads();
            for (uint32_t size = 2; size <= mp; size <<= 1) {
                for (uint32_t st = size >> 1; st > 0; st >>= 1) {
                    for (uint32_t q = tid; q < mp / 2; q += kClsThreads) {
                        const uint32_t lo = 2 * q - (q & (st - 1)), hi = lo + st;
                        const bool up = (lo & size) == 0;
                        const uint64_t ka = S.key[lo], kb = S.key[hi];
                        const uint16_t va = S.val[lo], vb = S.val[hi];
                        if (kv_less(kb, vb, ka, va) == up) { S.key[lo] = kb; S.key[hi] = ka; S.val[lo] = vb; S.val[hi] = va; }
                    }
                    __syncthreads();
                }
            }
            if (warp == 0) {  // prefix max of end in sorted order
                const uint32_t per = (m + 31) / 32;
                const uint32_t b = lane * per, e = min(b + per, m);
                uint64_t run = 0;
                for (uint32_t q = b; q < e; ++q) run = max(run, S.end[S.val[q]]);
                uint64_t incl = run;
                for (int d = 1; d < 32; d <<= 1) {
                    const uint64_t y = __shfl_up_sync(0xffffffffu, incl, d);
                    if (lane >= d) incl = max(incl, y);
                }
                uint64_t acc = __shfl_up_sync(0xffffffffu, incl, 1);
                if (lane == 0) acc = 0;
                for (uint32_t q = b; q < e; ++q) { acc = max(acc, S.end[S.val[q]]); S.pmax[q] = acc; }
            }
            __syncthreads();
#pragma unroll
            for (int k = 0; k < kWordsPerThread; ++k) {
                if (!cand[k] || hit[k]) continue;
                const uint64_t x = w[k];
                uint32_t lo = 0, hi = m;  // count of keys <= x
                while (lo < hi) { uint32_t mid = (lo + hi) >> 1; if (S.key[mid] <= x) lo = mid + 1; else hi = mid; }
                for (int q = (int)lo - 1; q >= 0 && S.pmax[q] > x; --q) {
                    const uint32_t u = S.val[q];
                    if (x - S.key[q] < S.end[u] - S.key[q] && S.ta[u] < t[k] && t[k] < S.tf[u]) {
                        hit[k] = true;
                        hid[k] = S.id[u];
                        hoff[k] = x - S.key[q];
                        break;
                    }
                }
            }
        }
        // I list: fence search in shared memory, then at most log2(stride) probes
#pragma unroll
        for (int k = 0; k < kWordsPerThread; ++k) {
            if (!cand[k] || hit[k] || nI == 0) continue;
            const uint64_t x = w[k];
            uint32_t lo = 0, hi = nf;  // count of fences <= x
            while (lo < hi) { uint32_t mid = (lo + hi) >> 1; if (S.fence[mid] <= x) lo = mid + 1; else hi = mid; }
            if (lo == 0) continue;
            uint32_t g0 = (lo - 1) * stride, g1 = min(g0 + stride, nI);
            uint32_t l2 = g0 + 1, h2 = g1;  // count of bases <= x within the group
            while (l2 < h2) { uint32_t mid = (l2 + h2) >> 1; if (p.d.i_base[mid] <= x) l2 = mid + 1; else h2 = mid; }
            const uint32_t kk = l2 - 1;
            const uint64_t base = stride == 1 ? S.fence[lo - 1] : p.d.i_base[kk];
            const IRest e = p.d.i_rest[kk];
            if (x < e.end && e.t_alloc < t[k]) {
                hit[k] = true;
                hid[k] = e.id;
                hoff[k] = x - base;
            }
        }
        // emission: mask words, per-(k,warp) counts, chunk prefix by look-back
        uint32_t bal[kWordsPerThread];
#pragma unroll
        for (int k = 0; k < kWordsPerThread; ++k) {
            bal[k] = __ballot_sync(0xffffffffu, hit[k]);
            const uint64_t mw = (cs + (uint64_t)k * kClsThreads + warp * 32) / 32;
            if (lane == 0) {
                S.cnt[k][warp] = __popc(bal[k]);
                if (mw < n_mask) a.mask[mw] = bal[k];
            }
        }
        __syncthreads();
        if (warp == 0) {
            // exclusive scan over (k, warp) in word order; 64 entries, 2 per lane
            const uint32_t e0 = S.cnt[(2 * lane) / kWarps][(2 * lane) % kWarps];
            const uint32_t e1 = S.cnt[(2 * lane + 1) / kWarps][(2 * lane + 1) % kWarps];
            const uint32_t pair = e0 + e1;
            uint32_t incl = pair;
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl += y;
            }
            const uint32_t excl = incl - pair;
            const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
            __syncwarp();
            S.cnt[(2 * lane) / kWarps][(2 * lane) % kWarps] = excl;
            S.cnt[(2 * lane + 1) / kWarps][(2 * lane + 1) % kWarps] = excl + e0;
            if (lane == 0) {
                unsigned long long prefix = 0;
                if (c == 0) {
                    st_release(&p.d.lookback[0], LB_PRE | total);
                } else {
                    st_release(&p.d.lookback[c], LB_AGG | total);
                    int64_t j = (int64_t)c - 1;
                    while (j >= 0) {
                        const unsigned long long v = ld_acquire(&p.d.lookback[j]);
                        if ((v & ~LB_VAL) == 0) { __nanosleep(20); continue; }
                        prefix += v & LB_VAL;
                        if (v & LB_PRE) break;
                        --j;
                    }
                    st_release(&p.d.lookback[c], LB_PRE | (prefix + total));
                }
                a.chunk_base[c] = (uint32_t)prefix;
                if (c + 1 == p.C) {
                    a.chunk_base[p.C] = (uint32_t)(prefix + total);
                    ctl->n_slots = prefix + total;
                }
                S.prefix = prefix;
            }
        }
        __syncthreads();
        const unsigned long long prefix = S.prefix;
        const uint32_t lt = lanemask_lt();
#pragma unroll
        for (int k = 0; k < kWordsPerThread; ++k) {
            if (!hit[k]) continue;
            const unsigned long long rank = prefix + S.cnt[k][warp] + __popc(bal[k] & lt);
            if (rank < a.capacity) a.slot[rank] = ((uint64_t)hid[k] << MEDUSA_OFF_BITS) | hoff[k];
        }
    }
}

// ----------------------------------------------------------------------------
// host side: per-device scratch, launches
struct Scratch {
    size_t cap_n = 0, cap_C = 0, cap_nb = 0, cap_c = 0, cap_b = 0;
    void* zero_region = nullptr;
    size_t zero_bytes = 0;
    Dev d{};
    std::vector<void*> bufs;
    Ctl* h_ctl = nullptr;
    int sm_count = 0, cls_blocks_per_sm = 0;
};
std::mutex g_mu;
std::vector<Scratch*> g_scratch;

template <class T>
cudaError_t grow(Scratch& s, T*& p, size_t elems) {
    T* q = nullptr;
    cudaError_t e = cudaMalloc(&q, std::max<size_t>(elems, 1) * sizeof(T));
    if (e != cudaSuccess) return e;
    p = q;
    s.bufs.push_back(q);
    return cudaSuccess;
}

void release(Scratch& s) {
    for (void* p : s.bufs) cudaFree(p);
    s.bufs.clear();
    if (s.zero_region) cudaFree(s.zero_region);
    s.zero_region = nullptr;
    s.cap_n = s.cap_C = s.cap_nb = s.cap_c = s.cap_b = 0;
}

cudaError_t ensure(Scratch& s, size_t n, size_t C, size_t nb, size_t need_c, size_t need_b) {
    if (n <= s.cap_n && C <= s.cap_C && nb <= s.cap_nb && need_c <= s.cap_c && need_b <= s.cap_b) return cudaSuccess;
    cudaDeviceSynchronize();
    release(s);
    const size_t N = std::max<size_t>(n, 1024), CC = std::max<size_t>(C, 64), NB = std::max<size_t>(nb, 64);
    const size_t RC = std::max<size_t>(need_c, 2 * N + 4 * CC), RB = std::max<size_t>(need_b, 3 * N);
    cudaError_t e;
    // zero region: Ctl | cnt_c fill_c [CC+1] | cnt_b fill_b [NB+1] | lookback [CC]
    s.zero_bytes = 256 + 2 * (CC + 1) * 4 + 2 * (NB + 1) * 4 + 8 * CC + 64;
    if ((e = cudaMalloc(&s.zero_region, s.zero_bytes)) != cudaSuccess) return e;
    char* z = (char*)s.zero_region;
    s.d.ctl = (Ctl*)z;
    size_t o = 256;
    s.d.cnt_c = (uint32_t*)(z + o); o += (CC + 1) * 4;
    s.d.fill_c = (uint32_t*)(z + o); o += (CC + 1) * 4;
    s.d.cnt_b = (uint32_t*)(z + o); o += (NB + 1) * 4;
    s.d.fill_b = (uint32_t*)(z + o); o += (NB + 1) * 4;
    o = (o + 7) & ~size_t(7);
    s.d.lookback = (unsigned long long*)(z + o);
    if ((e = grow(s, s.d.tmin, CC)) || (e = grow(s, s.d.tmax, CC)) || (e = grow(s, s.d.jf, CC)) ||
        (e = grow(s, s.d.jl, CC)) || (e = grow(s, s.d.rng, N)) || (e = grow(s, s.d.off_c, CC + 1)) ||
        (e = grow(s, s.d.off_b, NB + 1)) || (e = grow(s, s.d.list_c, RC)) || (e = grow(s, s.d.list_b, RB)) ||
        (e = grow(s, s.d.sk0, N)) || (e = grow(s, s.d.sk1, N)) || (e = grow(s, s.d.sv0, N)) ||
        (e = grow(s, s.d.sv1, N)) || (e = grow(s, s.d.i_base, N)) || (e = grow(s, s.d.i_rest, N)) ||
        (e = grow(s, s.d.fence, (size_t)kFenceCap)))
        return e;
    s.d.cap_c = RC;
    s.d.cap_b = RB;
    s.cap_n = N; s.cap_C = CC; s.cap_nb = NB; s.cap_c = RC; s.cap_b = RB;
    return cudaSuccess;
}

}  // namespace

medusa_status run_materialize(const MaterializeArgs& a, uint64_t* n_slots, cudaStream_t stream,
                              cudaError_t* cuda_err) {
    *n_slots = 0;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    std::lock_guard<std::mutex> lk(g_mu);
    if ((int)g_scratch.size() <= dev) g_scratch.resize(dev + 1, nullptr);
    if (!g_scratch[dev]) g_scratch[dev] = new Scratch();
    Scratch& s = *g_scratch[dev];
    if (!s.h_ctl) {
        if ((e = cudaMallocHost(&s.h_ctl, sizeof(Ctl))) != cudaSuccess) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
        cudaDeviceGetAttribute(&s.sm_count, cudaDevAttrMultiProcessorCount, dev);
        cudaFuncSetAttribute(k_classify, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(ClsShared));
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&s.cls_blocks_per_sm, k_classify, kClsThreads,
                                                      sizeof(ClsShared));
        if (s.cls_blocks_per_sm < 1) s.cls_blocks_per_sm = 1;
    }
    const uint64_t n = a.n_alloc;
    const uint32_t C = (uint32_t)((a.n_words + kChunkWords - 1) / kChunkWords);
    const uint32_t nb = (uint32_t)((n + kAblk - 1) / kAblk);
    size_t need_c = 0, need_b = 0;
    for (int attempt = 0; attempt < 3; ++attempt) {
        if ((e = ensure(s, n, C, nb, need_c, need_b)) != cudaSuccess) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
        P p{a, s.d, C, nb};
        if ((e = cudaMemsetAsync(s.zero_region, 0, s.zero_bytes, stream)) != cudaSuccess) break;
        if (C == 0 && (e = cudaMemsetAsync(a.chunk_base, 0, sizeof(uint32_t), stream)) != cudaSuccess) break;
        const uint32_t T = 256;
        {
            const uint64_t work = std::max<uint64_t>((uint64_t)a.n_nodes + 1, C);
            TimedLaunch tl("mat_nodes_chunks", stream);
            k_nodes_chunks<<<(unsigned)((work + T - 1) / T), T, 0, stream>>>(p);
        }
        if (n) {
            TimedLaunch tl("mat_allocs", stream);
            k_allocs<<<(unsigned)((n + T - 1) / T), T, 0, stream>>>(p);
        }
        {
            TimedLaunch tl("mat_scan", stream);
            k_scan<<<1, 1024, 0, stream>>>(p);
        }
        if (n) {
            TimedLaunch tl("mat_scatter", stream);
            k_scatter<<<(unsigned)((n + T - 1) / T), T, 0, stream>>>(p);
        }
        if (n) {
            const unsigned tiles = (unsigned)((n + kSortTile - 1) / kSortTile);
            {
                TimedLaunch tl("mat_sort_tile", stream);
                k_sort_tile<<<tiles, 1024, 0, stream>>>(s.d.ctl, s.d.sk0, s.d.sv0, s.d.sk1, s.d.sv1);
            }
            uint64_t *ki = s.d.sk1, *ko = s.d.sk0;
            uint32_t *vi = s.d.sv1, *vo = s.d.sv0;
            for (uint64_t width = kSortTile; width < n; width *= 2) {
                TimedLaunch tl("mat_merge", stream);
                k_merge<<<tiles, 256, 0, stream>>>(s.d.ctl, ki, vi, ko, vo, (uint32_t)width);
                std::swap(ki, ko);
                std::swap(vi, vo);
            }
            TimedLaunch tl("mat_build_i", stream);
            k_build_i<<<(unsigned)((n + T - 1) / T), T, 0, stream>>>(p, ki, vi);
        }
        if (n) {
            TimedLaunch tl("mat_check", stream);
            k_check<<<nb, kAblk, 0, stream>>>(p);
        }
        if (C) {
            const unsigned grid = (unsigned)std::min<uint64_t>(C, (uint64_t)s.sm_count * s.cls_blocks_per_sm);
            TimedLaunch tl("mat_classify", stream);
            k_classify<<<grid, kClsThreads, sizeof(ClsShared), stream>>>(p);
        }
        if ((e = cudaGetLastError()) != cudaSuccess) break;
        if ((e = cudaMemcpyAsync(s.h_ctl, s.d.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, stream)) != cudaSuccess) break;
        if ((e = cudaStreamSynchronize(stream)) != cudaSuccess) break;
        const Ctl h = *s.h_ctl;
        if (h.status & ST_INVALID) return MEDUSA_ERR_INVALID_ARG;
        if (h.status & ST_TRACE) return MEDUSA_ERR_TRACE;
        if (h.status & ST_OVERFLOW) {  // registration lists larger than guessed: size exactly, rerun
            need_c = h.need_c;
            need_b = h.need_b;
            continue;
        }
        *n_slots = h.n_slots;
        return h.n_slots > a.capacity ? MEDUSA_ERR_CAPACITY : MEDUSA_OK;
    }
    if (e != cudaSuccess) { *cuda_err = e; return MEDUSA_ERR_CUDA; }
    *cuda_err = cudaErrorUnknown;
    return MEDUSA_ERR_CUDA;
}

}  // namespace medusa
