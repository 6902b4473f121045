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
//   * one CTA of 256 threads per 2048-word chunk.  The chunk's 16 KB of words
//     move HBM -> shared memory -> HBM with the TMA engine (cp.async.bulk load
//     completing on an mbarrier, cp.async.bulk store from shared memory), so no
//     thread holds image words in registers and ~17 KB of shared memory and ~30
//     registers per CTA let 8 CTAs share an SM;
//   * the chunk's records are the contiguous range [chunk_base[c],
//     chunk_base[c+1]), known after one load.  Work is per record, not per
//     word: thread r loads record r (coalesced), gathers old_base / new_base /
//     new_size of its allocation (L2-resident, 24 B per allocation), finds its
//     word as the (r - prefix)-th set bit of one mask word (__fns over a 64-entry
//     shared popcount prefix), validates and rewrites the word in shared memory;
//   * gather tasks (2048 nodes each) are appended to the same grid;
//   * validation failures (rare) go to the report with atomics; a one-thread
//     kernel initializes the report first, so CTAs need no fence or ticket.
// Images whose base or length break TMA's 16-byte granularity use plain loads and
// stores through the same shared buffer.
#include <algorithm>

#include "common.cuh"

namespace medusa {
namespace {

constexpr int kTaskWords = MEDUSA_CHUNK_WORDS;  // 2048
constexpr int kThreads = 256;
constexpr int kMaskPerTask = kTaskWords / 32;   // 64
constexpr int kNodesPerTask = 2048;

__global__ void report_init(medusa_report* r) {
    r->n_bad_slot = 0;
    r->first_bad_word = ~0ull;
    r->n_bad_id = 0;
    r->n_bad_range = 0;
    r->n_stale = 0;
    r->n_bad_func = 0;
    r->first_bad_node = ~0ull;
    r->reserved = 0;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

constexpr int kStages = 3;
constexpr int kRecCap = 768;                  // records per stage delivered by TMA (else loaded directly)
constexpr int kConsumers = kThreads;          // 8 consumer warps
constexpr int kBlock = kConsumers + 32;       // + 1 producer warp

struct __align__(128) Stage {
    uint64_t words[kTaskWords];   // TMA in -> rewritten -> TMA out (16 KB)
    uint64_t recs[kRecCap + 2];   // the chunk's records from an even index (TMA)
    uint32_t mask[kMaskPerTask];  // TMA
    uint32_t pre[kMaskPerTask];
    uint32_t chunk, n, rec0, nrec;
    uint32_t flags;               // 1: words by TMA, 2: mask by TMA, 4: records by TMA
    uint32_t rec_skew;            // rec0 - first record delivered
};

__device__ __forceinline__ void mbar_wait(uint32_t mb, uint32_t parity) {
    uint32_t ready = 0;
    while (!ready) {
        asm volatile("{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2; selp.u32 %0, 1, 0, P; }"
                     : "=r"(ready) : "r"(mb), "r"(parity) : "memory");
    }
}
__device__ __forceinline__ void tma_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t mb) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(dst), "l"(src), "r"(bytes), "r"(mb) : "memory");
}
__device__ __forceinline__ void consumer_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kConsumers) : "memory"); }

// Warp-specialized persistent CTAs.  The producer warp (one lane) owns every TMA
// transfer: for chunk c = blockIdx.x + k*G it fills stage k % kStages with the
// chunk's words, mask words and records (one mbarrier with the byte count), and
// once the consumers signal the stage done it writes the words back with a TMA
// bulk store and refills the stage.  The 8 consumer warps only gather base-table
// entries, locate and rewrite slot words in shared memory.
__global__ void __launch_bounds__(kBlock, 3)
restore_kernel(RestoreArgs a, uint32_t n_word_tasks, uint32_t word_ctas, uint32_t n_node_tasks) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Stage* st = reinterpret_cast<Stage*>(smem_raw);
    __shared__ __align__(8) unsigned long long s_full[kStages], s_done[kStages];

    const uint32_t tid = threadIdx.x;
    unsigned long long* rep = reinterpret_cast<unsigned long long*>(a.report);

    if (blockIdx.x >= word_ctas) {  // kernel-address fill
        const uint32_t task = blockIdx.x - word_ctas;
        if (task >= n_node_tasks || tid >= kThreads) return;
        const uint64_t j0 = (uint64_t)task * kNodesPerTask;
        uint32_t n_bad = 0;
        uint64_t first = ~0ull;
#pragma unroll
        for (int k = 0; k < kNodesPerTask / kThreads; ++k) {
            const uint64_t j = j0 + tid + k * kThreads;
            if (j < a.n_nodes) {
                const uint32_t f = a.func_id[j];
                uint64_t addr = 0;
                if (f < a.n_func) addr = __ldg(a.table + f);
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
        return;
    }

    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&s_full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&s_done[s])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const uint32_t n_mine = n_word_tasks > blockIdx.x ? (n_word_tasks - blockIdx.x + word_ctas - 1) / word_ctas : 0;
    const uint64_t n_mask = (a.n_words + 31) / 32;
    const uint64_t n_rec_total = a.n_slots;

    if (tid >= kConsumers) {
        // ------------------------------------------------------------ producer
        if (tid != kConsumers) return;
        const bool aligned = ((reinterpret_cast<uintptr_t>(a.src) | reinterpret_cast<uintptr_t>(a.dst)) & 15) == 0;
        {  // warm L2 with this CTA's share of the replayed base table (gathered per record)
            const uint64_t bytes = (uint64_t)a.n_alloc * 8;
            const uint64_t per = ((bytes + word_ctas - 1) / word_ctas + 15) & ~15ull;
            const uint64_t b0 = (uint64_t)blockIdx.x * per;
            if (b0 < bytes) {
                const uint32_t len = (uint32_t)((min(b0 + per, bytes) - b0 + 15) & ~15ull);
                const uint64_t* arrs[3] = {a.new_size, a.old_base, a.new_base};
                for (int q = 0; q < 3; ++q) {
                    const char* base = reinterpret_cast<const char*>(arrs[q]);
                    if ((reinterpret_cast<uintptr_t>(base) & 15) == 0 && b0 + len <= ((bytes + 15) & ~15ull))
                        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(base + b0), "r"(len) : "memory");
                }
            }
        }
        auto store_stage = [&](int s) {  // words of the chunk held in stage s back to HBM
            Stage& S = st[s];
            if (S.flags & 1) {
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                             ::"l"(a.dst + (uint64_t)S.chunk * kTaskWords),
                             "r"((uint32_t)__cvta_generic_to_shared(S.words)), "r"(S.n * 8) : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
        };
        for (uint32_t k = 0; k < n_mine + kStages; ++k) {
            const int s = k % kStages;
            Stage& S = st[s];
            if (k >= kStages) {  // the stage's previous chunk: wait for the consumers, write it back
                mbar_wait((uint32_t)__cvta_generic_to_shared(&s_done[s]), ((k / kStages) - 1) & 1);
                store_stage(s);
                asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            }
            if (k >= n_mine) continue;
            const uint32_t c = blockIdx.x + k * word_ctas;
            const uint64_t ws = (uint64_t)c * kTaskWords;
            const uint32_t n = (uint32_t)min((uint64_t)kTaskWords, a.n_words - ws);
            const uint32_t r0 = a.chunk_base[c], r1 = a.chunk_base[c + 1];
            const uint32_t nrec = r1 > r0 ? r1 - r0 : 0;
            uint32_t flags = 0, bytes = 0;
            if (aligned && n % 2 == 0) { flags |= 1; bytes += n * 8; }
            const uint64_t m0 = (uint64_t)c * kMaskPerTask;
            if (m0 + kMaskPerTask <= n_mask && ((reinterpret_cast<uintptr_t>(a.mask + m0) & 15) == 0)) {
                flags |= 2;
                bytes += kMaskPerTask * 4;
            }
            const uint64_t e0 = r0 & ~1ull, e1 = ((uint64_t)r0 + nrec + 1) & ~1ull;  // even-aligned record span
            const bool rec_ok = nrec > 0 && nrec <= kRecCap && e1 <= min(n_rec_total, a.slot_capacity) &&
                                ((reinterpret_cast<uintptr_t>(a.slot) & 15) == 0);
            if (rec_ok) { flags |= 4; bytes += (uint32_t)(e1 - e0) * 8; }
            S.chunk = c; S.n = n; S.rec0 = r0; S.nrec = nrec; S.flags = flags; S.rec_skew = (uint32_t)(r0 - e0);
            const uint32_t mb = (uint32_t)__cvta_generic_to_shared(&s_full[s]);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(bytes) : "memory");
            if (flags & 1) tma_load((uint32_t)__cvta_generic_to_shared(S.words), a.src + ws, n * 8, mb);
            if (flags & 2) tma_load((uint32_t)__cvta_generic_to_shared(S.mask), a.mask + m0, kMaskPerTask * 4, mb);
            if (flags & 4) tma_load((uint32_t)__cvta_generic_to_shared(S.recs), a.slot + e0, (uint32_t)(e1 - e0) * 8, mb);
        }
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        return;
    }

    // -------------------------------------------------------------- consumers
    uint32_t n_id = 0, n_rg = 0, n_st = 0;
    uint64_t first = ~0ull;
    for (uint32_t k = 0; k < n_mine; ++k) {
        const int s = k % kStages;
        Stage& S = st[s];
        mbar_wait((uint32_t)__cvta_generic_to_shared(&s_full[s]), (k / kStages) & 1);
        const uint32_t c = S.chunk, n = S.n, flags = S.flags, nrec = S.nrec;
        const uint64_t ws = (uint64_t)c * kTaskWords;
        const uint64_t rec0 = S.rec0;
        if (!(flags & 1))
            for (uint32_t q = tid; q < n; q += kConsumers) S.words[q] = ld_stream(a.src + ws + q);
        if (!(flags & 2) && tid < kMaskPerTask) {
            const uint64_t mw = (uint64_t)c * kMaskPerTask + tid;
            S.mask[tid] = mw < n_mask ? a.mask[mw] : 0u;
        }
        if (!(flags & 2)) consumer_sync();
        if (tid < 32) {  // exclusive prefix of the 64 mask popcounts
            const uint32_t p0 = __popc(S.mask[2 * tid]), p1 = __popc(S.mask[2 * tid + 1]);
            uint32_t incl = p0 + p1;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (tid >= d) incl += y;
            }
            S.pre[2 * tid] = incl - p0 - p1;
            S.pre[2 * tid + 1] = incl - p1;
        }
        const uint32_t n_rec_c = min(nrec, (uint32_t)kTaskWords);
        // records, two per thread per round: gather, (prefix ready) locate, rewrite
        for (uint32_t rb = 0; rb < max(n_rec_c, 1u); rb += 2 * kConsumers) {
            uint64_t exp[2], nv[2];
            uint32_t kind[2];  // 0 ok, 1 bad id, 2 bad range, 3 none
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                const uint32_t r = rb + tid + u * kConsumers;
                kind[u] = 3;
                exp[u] = nv[u] = 0;
                if (r < n_rec_c) {
                    kind[u] = 1;
                    const uint64_t kk = rec0 + r;
                    if (kk < n_rec_total) {
                        const uint64_t rec = (flags & 4) ? S.recs[S.rec_skew + r] : a.slot[kk];
                        const uint64_t id = rec >> MEDUSA_OFF_BITS;
                        const uint64_t off = rec & kOffMask;
                        if (id < a.n_alloc) {
                            const uint64_t sz = __ldg(a.new_size + id);
                            const uint64_t ob = __ldg(a.old_base + id);
                            const uint64_t nb = __ldg(a.new_base + id);
                            if (off < sz) {
                                kind[u] = 0;
                                exp[u] = ob + off;
                                nv[u] = nb + off;
                            } else {
                                kind[u] = 2;
                            }
                        }
                    }
                }
            }
            if (rb == 0) consumer_sync();  // prefix (and directly loaded words) ready
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                if (kind[u] == 3) continue;
                const uint32_t r = rb + tid + u * kConsumers;
                uint32_t lo = 0, hi = kMaskPerTask;  // mask word m with pre[m] <= r < pre[m] + popc
                while (hi - lo > 1) { const uint32_t mid = (lo + hi) >> 1; if (S.pre[mid] <= r) lo = mid; else hi = mid; }
                const uint32_t bit = __fns(S.mask[lo], 0, r - S.pre[lo] + 1);
                const uint32_t q = lo * 32 + bit;
                bool bad = true;
                if (bit >= 32 || q >= n) {
                    ++n_id;  // more records than mask bits: nothing to apply
                } else if (kind[u] == 0) {
                    if (S.words[q] == exp[u]) { S.words[q] = nv[u]; bad = false; }
                    else ++n_st;
                } else if (kind[u] == 1) {
                    ++n_id;
                } else {
                    ++n_rg;
                }
                if (bad) first = min(first, ws + (q < n ? q : 0));
            }
        }
        // slots the mask shows beyond the table's records have nothing to apply
        if (tid == 0 && nrec > (uint32_t)kTaskWords) n_id += nrec - kTaskWords;
        if (!(flags & 1)) {
            consumer_sync();
            for (uint32_t q = tid; q < n; q += kConsumers) st_stream(a.dst + ws + q, S.words[q]);
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // rewrites visible to the TMA store
        consumer_sync();
        if (tid == 0)
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&s_done[s]))
                         : "memory");
    }
    if (n_id | n_rg | n_st) {
        atomicAdd(rep + 0, (unsigned long long)(n_id + n_rg + n_st));
        atomicMin(rep + 1, (unsigned long long)first);
        if (n_id) atomicAdd(rep + 2, (unsigned long long)n_id);
        if (n_rg) atomicAdd(rep + 3, (unsigned long long)n_rg);
        if (n_st) atomicAdd(rep + 4, (unsigned long long)n_st);
    }
}

}  // namespace

cudaError_t launch_restore(const RestoreArgs& a, cudaStream_t stream) {
    static int sm_count = 0;
    if (!sm_count) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sm_count, cudaDevAttrMultiProcessorCount, dev);
        if (sm_count <= 0) sm_count = 148;
        cudaFuncSetAttribute(restore_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kStages * (int)sizeof(Stage));
    }
    const uint32_t n_word_tasks = (uint32_t)((a.n_words + kTaskWords - 1) / kTaskWords);
    const uint32_t n_node_tasks = a.func_id ? (a.n_nodes + kNodesPerTask - 1) / kNodesPerTask : 0;
    const uint32_t word_ctas = std::min<uint32_t>(n_word_tasks, (uint32_t)sm_count * 3);
    {
        TimedLaunch tl("restore_report_init", stream);
        report_init<<<1, 1, 0, stream>>>(a.report);
    }
    if (word_ctas + n_node_tasks) {
        TimedLaunch tl("restore", stream);
        restore_kernel<<<word_ctas + n_node_tasks, kBlock, kStages * sizeof(Stage), stream>>>(a, n_word_tasks, word_ctas,
                                                                                              n_node_tasks);
    }
    return cudaGetLastError();
}

}  // namespace medusa
