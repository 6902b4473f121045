// K3 relocate+validate and K4 kernel-address gather, fused into one launch.
//
// Replay-based data pointer restoration (§4.2): every slot
// (word g, allocation i, offset off) of the indirect-index-pointer table becomes
// new_base[i] + off, after the per-slot validation of DESIGN.md R-Q8;
// constants are copied.  Kernel-address fill:
// func_out[j] = table[func_id[j]].
//
// The pass is HBM-bound: per word it reads 8 B and writes 8 B; the mask adds
// 1/8 B, each slot record 8 B (about 18% of words are slots).  Design (B200):
//   * one CTA of 256 threads per two consecutive 2048-word chunks (one chunk per
//     CTA for images under two chunks per SM, e.g. a single model's set, so the
//     grid still spreads over the SMs).  The chunk's 16 KB of words
//     move HBM -> shared memory -> HBM with the TMA engine (cp.async.bulk load
//     completing on an mbarrier, cp.async.bulk store from shared memory), so no
//     thread holds image words in registers; ~17 KB of shared memory and ~35
//     registers per CTA let 6-7 CTAs share an SM.  (Measured alternatives --
//     128-thread CTAs, persistent CTAs with a 2-stage ring, a warp-specialized
//     TMA producer over a 3-stage ring -- were slower: tools/microbench_restore.cu
//     and DESIGN.md §5);
//   * thread 0 also asks the TMA engine to prefetch this CTA's slice of the
//     three base-table arrays into L2 (cp.async.bulk.prefetch.L2), so the
//     per-record gathers of every CTA hit L2;
//   * the chunk's records are the contiguous range [chunk_base[c],
//     chunk_base[c+1]), known after one load.  Work is per record, not per
//     word: thread r loads record r (coalesced), gathers old_base / new_base /
//     new_size of its allocation (L2-resident, 24 B per allocation), finds its
//     word as the (r - prefix)-th set bit of one mask word (nth_set_bit over a 64-entry
//     shared popcount prefix), validates and rewrites the word in shared memory;
//   * gather tasks (2048 nodes each) are appended to the same grid;
//   * validation failures (rare) go to the report with atomics; a one-thread
//     kernel initializes the report first, so CTAs need no fence or ticket.
// Images whose base or length break TMA's 16-byte granularity use plain loads and
// stores through the same shared buffer.
#include "common.cuh"

namespace medusa {
namespace {

constexpr int kTaskWords = MEDUSA_CHUNK_WORDS;  // 2048
constexpr int kThreads = 256;
constexpr int kMaskPerTask = kTaskWords / 32;   // 64
constexpr int kNodesPerTask = 2048;

MEDUSA_TL_DEFINE

__global__ void report_init(medusa_report* r) {
    const unsigned long long tl0 = TL_NOW();
    if (MEDUSA_EARLY_TRIGGER) pdl_trigger();  // (the restore waits before it reads the table)
    pdl_wait();  // the previous user of the report may still read it
    if (!MEDUSA_EARLY_TRIGGER) pdl_trigger();
    r->n_bad_slot = 0;
    r->first_bad_word = ~0ull;
    r->n_bad_id = 0;
    r->n_bad_range = 0;
    r->n_stale = 0;
    r->n_bad_func = 0;
    r->first_bad_node = ~0ull;
    r->n_bad_chunk = 0;
    TL_REC(6, 0, tl0);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

// Kernel-address fill of 2048 nodes (gather task gt): func_out[j] =
// table[func_id[j]], unresolved ids counted.
__device__ __forceinline__ void gather_role(const RestoreArgs& a, uint32_t gt, unsigned long long* rep) {
    const uint32_t tid = threadIdx.x;
    const uint64_t j0 = (uint64_t)gt * kNodesPerTask;
    uint32_t n_bad = 0;
    uint64_t first = ~0ull;
    constexpr int kPer = kNodesPerTask / kThreads;
    uint32_t f[kPer];
#pragma unroll
    for (int k = 0; k < kPer; ++k) {  // the kernel ids (an input) before the wait
        const uint64_t j = j0 + tid + k * kThreads;
        f[k] = j < a.n_nodes ? a.func_id[j] : 0u;
    }
    // the kernel table may have been written by a kernel two or more launches back
    // (k_table_copy; the tail of a call triggers its successors early: common.cuh)
    pdl_wait();
    pdl_trigger();
#pragma unroll
    for (int k = 0; k < kPer; ++k) {
        const uint64_t j = j0 + tid + k * kThreads;
        if (j < a.n_nodes) {
            uint64_t addr = 0;
            if (f[k] < a.n_func) addr = __ldg(a.table + f[k]);
            if (addr == 0) {
                ++n_bad;
                first = min(first, j);
            }
            a.func_out[j] = addr;
        }
    }
    if (n_bad) {
        atomicAdd(rep + 5, (unsigned long long)n_bad);
        atomicMin(rep + 6, (unsigned long long)first);
    }
}

// Table view of the CTA's CPB chunks (DESIGN.md R-TABLE): the mask words (bits of
// words past n_words cleared), their popcount prefix (pre[kMask] = the CTA's
// slot count), the chunk_base entries, and which chunks are consistent -- chunk
// h is iff its record range [cb[h], cb[h+1]) holds exactly as many records as
// its mask has bits.  The i-th set bit of a consistent chunk pairs with record
// cb[h] + i; an inconsistent chunk is copied unchanged and counted (n_bad_chunk).
template <int CPB>
struct TableView {
    static constexpr uint32_t kMask = CPB * kMaskPerTask;
    uint32_t mask[kMask];
    uint32_t pre[kMask + 1];
    uint32_t cb[CPB + 1];
    uint32_t ok;  // bit h: chunk h consistent
};

// (whole CTA) the mask words and the chunk_base entries; ends with a barrier
template <int CPB>
__device__ __forceinline__ void table_load(const RestoreArgs& a, uint32_t task, TableView<CPB>& T) {
    constexpr uint32_t kMask = TableView<CPB>::kMask;
    const uint64_t n_mask = (a.n_words + 31) / 32;
    const uint64_t mw0 = (uint64_t)task * kMask;
    const uint64_t n_chunks = (a.n_words + kTaskWords - 1) / kTaskWords;
    for (uint32_t m = threadIdx.x; m < kMask; m += kThreads) {
        const uint64_t mw = mw0 + m;
        uint32_t v = 0;
        if (mw < n_mask) {
            v = a.mask[mw];
            const uint64_t left = a.n_words - mw * 32;  // words of this mask word inside the image
            if (left < 32) v &= (1u << left) - 1u;
        }
        T.mask[m] = v;
    }
    if (threadIdx.x >= kThreads - (CPB + 1)) {  // chunks past the image read the total: 0 records, 0 bits
        const uint32_t h = threadIdx.x - (kThreads - (CPB + 1));
        T.cb[h] = a.chunk_base[min((uint64_t)task * CPB + h, n_chunks)];
    }
    __syncthreads();
}

// (warp 0) exclusive popcount prefix of the mask words and the consistency bits
template <int CPB>
__device__ __forceinline__ void table_prefix(TableView<CPB>& T) {
    constexpr int kPer = TableView<CPB>::kMask / 32;
    const uint32_t lane = threadIdx.x & 31;
    uint32_t pc[kPer], incl = 0;
#pragma unroll
    for (int j = 0; j < kPer; ++j) { pc[j] = __popc(T.mask[kPer * lane + j]); incl += pc[j]; }
    const uint32_t own = incl;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
        if (lane >= (uint32_t)d) incl += y;
    }
    uint32_t run = incl - own;
#pragma unroll
    for (int j = 0; j < kPer; ++j) { T.pre[kPer * lane + j] = run; run += pc[j]; }
    if (lane == 31) T.pre[TableView<CPB>::kMask] = incl;
    __syncwarp();
    if (lane == 0) {
        uint32_t ok = 0;
#pragma unroll
        for (int h = 0; h < CPB; ++h) {
            const uint32_t bits = T.pre[(h + 1) * kMaskPerTask] - T.pre[h * kMaskPerTask];
            if (T.cb[h + 1] >= T.cb[h] && T.cb[h + 1] - T.cb[h] == bits) ok |= 1u << h;
        }
        T.ok = ok;
    }
}

// record index of the CTA's r-th slot bit; false if its chunk is inconsistent
template <int CPB>
__device__ __forceinline__ bool table_rec(const TableView<CPB>& T, uint32_t r, uint64_t& k) {
    const uint32_t h = (CPB == 2 && r >= T.pre[kMaskPerTask]) ? 1u : 0u;
    k = (uint64_t)T.cb[h] + (r - T.pre[h * kMaskPerTask]);
    return (T.ok >> h) & 1u;
}

// word (in the CTA) of the r-th slot bit, r < pre[kMask]
template <int CPB>
__device__ __forceinline__ uint32_t table_word(const TableView<CPB>& T, uint32_t r) {
    uint32_t lo = 0;  // last mask word m with pre[m] <= r (pre[0] = 0): binary lifting, no branches
#pragma unroll
    for (uint32_t st = TableView<CPB>::kMask / 2; st > 0; st >>= 1) lo += T.pre[lo + st] <= r ? st : 0u;
    MCHECK(lo < TableView<CPB>::kMask && r >= T.pre[lo] && r - T.pre[lo] < (uint32_t)__popc(T.mask[lo]));
    return lo * 32 + nth_set_bit(T.mask[lo], r - T.pre[lo]);
}

// record k -> kind (0 ok, 1 bad id / missing record, 2 bad range), expected source
// word and relocated value (DESIGN.md R-Q8, R-TABLE)
__device__ __forceinline__ uint32_t load_rec(const RestoreArgs& a, uint64_t k, uint64_t& exp, uint64_t& nv) {
    exp = nv = 0;
    if (k >= a.n_slots) return 1;  // no record: the caller's slot count ends before it
    const uint64_t rec = a.slot[k];
    const uint64_t id = rec >> MEDUSA_OFF_BITS;
    const uint64_t off = rec & kOffMask;
    if (id >= a.n_alloc) return 1;
    const uint64_t sz = __ldg(a.new_size + id);
    const uint64_t ob = __ldg(a.old_base + id);
    const uint64_t nb = __ldg(a.new_base + id);
    if (off >= sz) return 2;
    exp = ob + off;
    nv = nb + off;
    return 0;
}

// the two halves of load_rec, for the in-place pass: the record load, then (once
// it has landed) the replay-table gathers
__device__ __forceinline__ uint64_t rec_load(const RestoreArgs& a, uint64_t k) {
    return k < a.n_slots ? a.slot[k] : 0ull;
}
__device__ __forceinline__ uint32_t rec_kind(const RestoreArgs& a, uint64_t k, uint64_t rec, uint64_t& exp,
                                             uint64_t& nv) {
    exp = nv = 0;
    if (k >= a.n_slots) return 1;
    const uint64_t id = rec >> MEDUSA_OFF_BITS;
    const uint64_t off = rec & kOffMask;
    if (id >= a.n_alloc) return 1;
    const uint64_t sz = __ldg(a.new_size + id);
    const uint64_t ob = __ldg(a.old_base + id);
    const uint64_t nb = __ldg(a.new_base + id);
    if (off >= sz) return 2;
    exp = ob + off;
    nv = nb + off;
    return 0;
}

__device__ __forceinline__ void report_add(unsigned long long* rep, uint32_t n_id, uint32_t n_rg, uint32_t n_st,
                                           uint64_t first, uint32_t n_chunk) {
    if (n_id | n_rg | n_st) {
        atomicAdd(rep + 0, (unsigned long long)(n_id + n_rg + n_st));
        atomicMin(rep + 1, (unsigned long long)first);
        if (n_id) atomicAdd(rep + 2, (unsigned long long)n_id);
        if (n_rg) atomicAdd(rep + 3, (unsigned long long)n_rg);
        if (n_st) atomicAdd(rep + 4, (unsigned long long)n_st);
    }
    if (n_chunk) atomicAdd(rep + 7, (unsigned long long)n_chunk);
}

#ifndef MEDUSA_RESTORE_PER
#define MEDUSA_RESTORE_PER 2
#endif
constexpr int kRestorePer2 = MEDUSA_RESTORE_PER;  // records per thread in flight per round, two-chunk CTAs (3 and 4:
                                                  //  a shorter apply phase, a longer first round: ALL10 restore
                                                  //  span +1.3 / +1.9 us, measured)
template <int CPB>
__global__ void __launch_bounds__(kThreads, (CPB == 1 ? 8 : 6))
restore_kernel(RestoreArgs a, uint32_t n_word_tasks, uint32_t n_tasks) {
    constexpr uint32_t kWords = CPB * kTaskWords;   // words of this CTA (CPB consecutive chunks)
    constexpr uint32_t kMask = CPB * kMaskPerTask;  // their mask words
    constexpr uint32_t kAllOk = (1u << CPB) - 1u;
    constexpr int kRestorePer = CPB == 2 ? kRestorePer2 : 2;
    __shared__ __align__(128) uint64_t s_words[kWords];
    __shared__ TableView<CPB> T;
    __shared__ __align__(8) unsigned long long s_mbar[CPB];

    const uint32_t tid = threadIdx.x;
    const uint32_t task = blockIdx.x;
    unsigned long long* rep = reinterpret_cast<unsigned long long*>(a.report);
    const unsigned long long tl0 = TL_NOW();
    unsigned long long tl_p = tl0;

    if (task < n_word_tasks) {
        const uint64_t ws = (uint64_t)task * kWords;
        const uint32_t n = (uint32_t)min((uint64_t)kWords, a.n_words - ws);
        const uint64_t* gsrc = a.src + ws;
        uint64_t* gdst = a.dst + ws;
        const bool tma = (((reinterpret_cast<uintptr_t>(gsrc) | reinterpret_cast<uintptr_t>(gdst)) & 15) == 0) &&
                         (n % 2 == 0);
        if (tid == 0) {  // warm L2 with this CTA's slice of the replayed base table
            const uint64_t bytes = (uint64_t)a.n_alloc * 8;
            const uint64_t per = ((bytes + n_word_tasks - 1) / n_word_tasks + 255) & ~255ull;
            const uint64_t b0 = (uint64_t)task * per;
            if (b0 < bytes) {
                const uint32_t len = (uint32_t)((min(b0 + per, bytes) - b0 + 15) & ~15ull);
                const uint64_t* arrs[3] = {a.new_size, a.old_base, a.new_base};
#pragma unroll
                for (int q = 0; q < 3; ++q) {
                    const char* base = reinterpret_cast<const char*>(arrs[q]);
                    if ((reinterpret_cast<uintptr_t>(base) & 15) == 0)
                        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(base + b0), "r"(len) : "memory");
                }
            }
        }
        // 1. the CTA's words: one bulk copy per chunk into shared memory (all issued
        //    at once); meanwhile the mask words and the record ranges.  (Issuing the
        //    copies after those small loads measured the same: their ~3 us is not
        //    queueing behind the bulk reads.)
        if (tid == 0 && tma) {
#pragma unroll
            for (int c = 0; c < CPB; ++c) {
                const uint32_t mb = smem_u32(&s_mbar[c]);
                asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
            }
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
#pragma unroll
            for (int c = 0; c < CPB; ++c) {
                const uint32_t q0 = c * kTaskWords;
                if (q0 >= n) break;
                const uint32_t nc = min(n - q0, kTaskWords);
                const uint32_t mb = smem_u32(&s_mbar[c]);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(nc * 8) : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(smem_u32(s_words + q0)), "l"(gsrc + q0), "r"(nc * 8), "r"(mb) : "memory");
            }
        }
        if (!tma)
            for (uint32_t q = tid; q < n; q += kThreads) s_words[q] = ld_stream(gsrc + q);
        pdl_wait();  // the table (the previous kernels' output) and the report are ready
        table_load<CPB>(a, task, T);
        TL_PHASE(7, 10, tl_p);  // mask + record range loaded
        // 2. popcount prefix and consistency (warp 0) while the other warps load the
        //    first records, assuming every chunk consistent (the normal case:
        //    record cb[0] + r for bit r); checked after the barrier
        if (tid < 32) table_prefix<CPB>(T);
        const uint32_t cb0 = T.cb[0];
        uint32_t n_bits = T.cb[CPB] >= cb0 ? min(T.cb[CPB] - cb0, kWords) : 0u;  // exact once verified
        // 3. records, kRestorePer per thread per round: load, gather, (after the prefix is
        //    ready) locate the word, validate and rewrite it in shared memory
        uint32_t n_id = 0, n_rg = 0, n_st = 0;
        uint64_t first = ~0ull;
        uint32_t ready_mask = tma ? 0u : ~0u;  // chunks whose words have landed
        bool fast = true;
        for (uint32_t rb = 0; rb < max(n_bits, 1u); rb += kRestorePer * kThreads) {
            uint64_t exp[kRestorePer], nv[kRestorePer];
            uint32_t kind[kRestorePer];  // 0 ok, 1 bad id, 2 bad range, 3 none
#pragma unroll
            for (int u = 0; u < kRestorePer; ++u) {
                const uint32_t r = rb + tid + u * kThreads;
                kind[u] = 3;
                exp[u] = nv[u] = 0;
                uint64_t k = (uint64_t)cb0 + r;
                if (r < n_bits && (fast || table_rec<CPB>(T, r, k))) kind[u] = load_rec(a, k, exp[u], nv[u]);
            }
            if (rb == 0) {
                __syncthreads();  // prefix and consistency ready
                TL_PHASE(7, 11, tl_p);  // first records + gathers in
                n_bits = T.pre[kMask];
                if (T.ok != kAllOk) {  // (rare) an inconsistent chunk: round 0 again, chunk by chunk
                    fast = false;
#pragma unroll
                    for (int u = 0; u < kRestorePer; ++u) {
                        const uint32_t r = tid + u * kThreads;
                        uint64_t k;
                        kind[u] = (r < n_bits && table_rec<CPB>(T, r, k)) ? load_rec(a, k, exp[u], nv[u]) : 3u;
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < kRestorePer; ++u) {
                if (kind[u] == 3) continue;
                const uint32_t r = rb + tid + u * kThreads;
                const uint32_t q = table_word<CPB>(T, r);
                const uint32_t c = q / kTaskWords;
                if (!((ready_mask >> c) & 1u)) {  // this chunk's words: wait for its bulk copy
                    const uint32_t mb = smem_u32(&s_mbar[c]);
                    uint32_t ready = 0;
                    while (!ready) {
                        asm volatile("{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], 0; selp.u32 %0, 1, 0, P; }"
                                     : "=r"(ready) : "r"(mb) : "memory");
                    }
                    ready_mask |= 1u << c;
                }
                bool bad = true;
                if (kind[u] == 0) {
                    if (s_words[q] == exp[u]) { s_words[q] = nv[u]; bad = false; }
                    else ++n_st;
                } else if (kind[u] == 1) {
                    ++n_id;
                } else {
                    ++n_rg;
                }
                if (bad) first = min(first, ws + q);
            }
        }
        // every chunk's bulk copy must have landed before its words go back out
        if (tid == 0 && tma) {
#pragma unroll
            for (int c = 0; c < CPB; ++c) {
                if ((ready_mask >> c) & 1u || c * kTaskWords >= n) continue;
                const uint32_t mb = smem_u32(&s_mbar[c]);
                uint32_t ready = 0;
                while (!ready) {
                    asm volatile("{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], 0; selp.u32 %0, 1, 0, P; }"
                                 : "=r"(ready) : "r"(mb) : "memory");
                }
            }
        }
        __syncthreads();
        TL_PHASE(7, 12, tl_p);  // all records applied (incl. waiting for the words)
        // 4. the CTA's words back to HBM
        if (tma) {
            if (tid == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
#pragma unroll
                for (int c = 0; c < CPB; ++c) {
                    const uint32_t q0 = c * kTaskWords;
                    if (q0 >= n) break;
                    const uint32_t nc = min(n - q0, kTaskWords);
                    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                                 ::"l"(gdst + q0), "r"(smem_u32(s_words + q0)), "r"(nc * 8) : "memory");
                }
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            }
        } else {
            for (uint32_t q = tid; q < n; q += kThreads) st_stream(gdst + q, s_words[q]);
        }
        TL_PHASE(7, 13, tl_p);  // bulk store issued and read out of shared memory
        pdl_trigger();
        report_add(rep, n_id, n_rg, n_st, first, tid == 0 ? __popc(kAllOk & ~T.ok) : 0u);
        TL_REC(7, 0, tl0);
    } else if (task < n_tasks) {
        gather_role(a, task - n_word_tasks, rep);
        TL_REC(7, 1, tl0);
    }
}

// In place (dst == src): only the slot words are read and written -- the words
// in between are constants that stay where they are.  One CTA per
// CPB chunks: mask words + record ranges, popcount prefix, then per record:
// load, gather, locate its word, read it, validate, write it back.  No word
// staging, so the pass moves ~8 B/slot of image instead of 16 B/word.
template <int CPB>
__global__ void __launch_bounds__(kThreads)
restore_inplace_kernel(RestoreArgs a, uint32_t n_word_tasks, uint32_t n_tasks) {
    constexpr uint32_t kWords = CPB * kTaskWords;
    constexpr uint32_t kMask = CPB * kMaskPerTask;
    constexpr uint32_t kAllOk = (1u << CPB) - 1u;
#ifndef MEDUSA_INPLACE_PER
#define MEDUSA_INPLACE_PER 2
#endif
    constexpr uint32_t kPer = MEDUSA_INPLACE_PER;  // records per thread per round
    __shared__ TableView<CPB> T;
    const uint32_t tid = threadIdx.x;
    const uint32_t task = blockIdx.x;
    unsigned long long* rep = reinterpret_cast<unsigned long long*>(a.report);
    const unsigned long long tl0 = TL_NOW();
    if (task < n_word_tasks) {
        const uint64_t ws = (uint64_t)task * kWords;
        pdl_wait();  // the table (the previous kernels' output) and the report are ready
        table_load<CPB>(a, task, T);
        if (tid < 32) table_prefix<CPB>(T);
        const uint32_t cb0 = T.cb[0];
        uint32_t n_bits = T.cb[CPB] >= cb0 ? min(T.cb[CPB] - cb0, kWords) : 0u;
        uint32_t n_id = 0, n_rg = 0, n_st = 0;
        uint64_t first = ~0ull;
        bool fast = true;
        // per round: the records (issued first), then -- independent of them -- each
        // slot word located from the mask and loaded, then the replay-table gathers
        // of the records: two dependent rounds, not three
        for (uint32_t rb = 0; rb < max(n_bits, 1u); rb += kPer * kThreads) {
            uint64_t rec[kPer], kk[kPer];
            bool has[kPer];
#pragma unroll
            for (int u = 0; u < kPer; ++u) {
                const uint32_t r = rb + tid + u * kThreads;
                kk[u] = (uint64_t)cb0 + r;
                has[u] = r < n_bits && (fast || table_rec<CPB>(T, r, kk[u]));
                rec[u] = has[u] ? rec_load(a, kk[u]) : 0ull;
            }
            if (rb == 0) {
                __syncthreads();  // prefix and consistency ready
                n_bits = T.pre[kMask];
                if (T.ok != kAllOk) {  // (rare) an inconsistent chunk: round 0 again, chunk by chunk
                    fast = false;
#pragma unroll
                    for (int u = 0; u < kPer; ++u) {
                        const uint32_t r = tid + u * kThreads;
                        has[u] = r < n_bits && table_rec<CPB>(T, r, kk[u]);
                        rec[u] = has[u] ? rec_load(a, kk[u]) : 0ull;
                    }
                }
            }
            uint32_t qs[kPer];
            uint64_t cur[kPer];
#pragma unroll
            for (int u = 0; u < kPer; ++u) {  // locate every word first, then load them together
                if (!has[u]) continue;
                qs[u] = table_word<CPB>(T, rb + tid + u * kThreads);
                cur[u] = ld_stream(a.src + ws + qs[u]);
            }
            uint64_t exp[kPer], nv[kPer];
            uint32_t kind[kPer];  // 0 ok, 1 bad id, 2 bad range, 3 none
#pragma unroll
            for (int u = 0; u < kPer; ++u) kind[u] = has[u] ? rec_kind(a, kk[u], rec[u], exp[u], nv[u]) : 3u;
#pragma unroll
            for (int u = 0; u < kPer; ++u) {
                if (kind[u] == 3) continue;
                const uint32_t q = qs[u];
                bool bad = true;
                if (kind[u] == 0) {
                    if (cur[u] == exp[u]) { st_stream(a.dst + ws + q, nv[u]); bad = false; }
                    else ++n_st;
                } else if (kind[u] == 1) {
                    ++n_id;
                } else {
                    ++n_rg;
                }
                if (bad) first = min(first, ws + q);
            }
        }
        pdl_trigger();
        report_add(rep, n_id, n_rg, n_st, first, tid == 0 ? __popc(kAllOk & ~T.ok) : 0u);
        TL_REC(7, 2, tl0);
    } else if (task < n_tasks) {
        gather_role(a, task - n_word_tasks, rep);
        TL_REC(7, 1, tl0);
    }
}

}  // namespace

#ifndef MEDUSA_RESTORE_CPB
#define MEDUSA_RESTORE_CPB 2
#endif
constexpr int kCPB = MEDUSA_RESTORE_CPB;  // chunks per restore CTA (out of place)
#ifndef MEDUSA_RESTORE_CPB_IP
#define MEDUSA_RESTORE_CPB_IP 2
#endif
constexpr int kCPBInPlace = MEDUSA_RESTORE_CPB_IP;  // chunks per restore CTA (in place)

cudaError_t launch_restore(const RestoreArgs& a, cudaStream_t stream) {
    const bool in_place = a.src == a.dst;
    int dev = 0, sm_count = 148;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sm_count, cudaDevAttrMultiProcessorCount, dev);
    // small images (a single model's graph set): one chunk per CTA, so the CTAs
    // spread over more SMs and each chain of dependent loads is half as long
    const bool small = (a.n_words + 2ull * kTaskWords - 1) / (2ull * kTaskWords) < (uint64_t)sm_count;
    const uint64_t cpb = small ? 1 : (in_place ? kCPBInPlace : kCPB);
    const uint32_t n_word_tasks = (uint32_t)((a.n_words + cpb * kTaskWords - 1) / (cpb * kTaskWords));
    const uint32_t n_node_tasks = a.func_id ? (a.n_nodes + kNodesPerTask - 1) / kNodesPerTask : 0;
    const uint32_t n_tasks = n_word_tasks + n_node_tasks;
    {
        TimedLaunch tl("restore_report_init", stream);
        cudaError_t e = launch_pdl(report_init, 1, 1, 0, stream, a.report);
        if (e != cudaSuccess) return e;
    }
    if (n_tasks) {
        TimedLaunch tl("restore", stream);
        cudaError_t e = in_place
            ? (small ? launch_pdl(restore_inplace_kernel<1>, n_tasks, kThreads, 0, stream, a, n_word_tasks, n_tasks)
                     : launch_pdl(restore_inplace_kernel<kCPBInPlace>, n_tasks, kThreads, 0, stream, a, n_word_tasks, n_tasks))
            : (small ? launch_pdl(restore_kernel<1>, n_tasks, kThreads, 0, stream, a, n_word_tasks, n_tasks)
                     : launch_pdl(restore_kernel<kCPB>, n_tasks, kThreads, 0, stream, a, n_word_tasks, n_tasks));
        if (e != cudaSuccess) return e;
    }
    return cudaGetLastError();
}

}  // namespace medusa

#ifdef MEDUSA_TIMELINE
extern "C" int medusa_tl_attach_res(void* buf, unsigned cap) {
    unsigned zero = 0;
    medusa::TlRec* b = static_cast<medusa::TlRec*>(buf);
    if (cudaMemcpyToSymbol(medusa::g_tl, &b, sizeof(b)) != cudaSuccess) return -1;
    if (cudaMemcpyToSymbol(medusa::g_tl_cap, &cap, sizeof(cap)) != cudaSuccess) return -1;
    return cudaMemcpyToSymbol(medusa::g_tl_n, &zero, sizeof(zero)) == cudaSuccess ? 0 : -1;
}
extern "C" unsigned medusa_tl_count_res() {
    unsigned n = 0;
    cudaMemcpyFromSymbol(&n, medusa::g_tl_n, sizeof(n));
    return n;
}
#endif
