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

struct __align__(128) Stage {
    uint64_t words[kTaskWords];  // TMA destination and source (16 KB)
    uint32_t mask[kMaskPerTask];
    uint32_t pre[kMaskPerTask];
    uint32_t rec0, nrec;
};

__device__ __forceinline__ void mbar_wait(uint32_t mb, uint32_t parity) {
    uint32_t ready = 0;
    while (!ready) {
        asm volatile("{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2; selp.u32 %0, 1, 0, P; }"
                     : "=r"(ready) : "r"(mb), "r"(parity) : "memory");
    }
}

// Persistent CTAs over chunks c = blockIdx.x, + gridWords, ...  Two stages: while
// chunk c is processed from stage b, the TMA engine brings chunk c+G's words into
// stage b^1, and its mask words, record range and first records arrive in registers.
__global__ void __launch_bounds__(kThreads, 4)
restore_kernel(RestoreArgs a, uint32_t n_word_tasks, uint32_t word_ctas, uint32_t n_node_tasks) {
    __shared__ __align__(128) Stage st[2];
    __shared__ __align__(8) unsigned long long s_mbar[2];

    const uint32_t tid = threadIdx.x;
    unsigned long long* rep = reinterpret_cast<unsigned long long*>(a.report);

    if (blockIdx.x >= word_ctas) {  // kernel-address fill
        const uint32_t task = blockIdx.x - word_ctas;
        if (task >= n_node_tasks) return;
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

    const uint64_t n_mask = (a.n_words + 31) / 32;
    const bool aligned = ((reinterpret_cast<uintptr_t>(a.src) | reinterpret_cast<uintptr_t>(a.dst)) & 15) == 0;
    auto chunk_n = [&](uint32_t c) { return (uint32_t)min((uint64_t)kTaskWords, a.n_words - (uint64_t)c * kTaskWords); };
    auto chunk_tma = [&](uint32_t c) { return aligned && (chunk_n(c) % 2 == 0); };
    const uint32_t mb0 = (uint32_t)__cvta_generic_to_shared(&s_mbar[0]);
    const uint32_t mb1 = (uint32_t)__cvta_generic_to_shared(&s_mbar[1]);

    // prefetch of chunk c into stage b: words by TMA; mask words / record range /
    // first records into registers (written to shared memory at the next step)
    uint32_t pf_mask = 0, pf_cb0 = 0, pf_cb1 = 0;
    auto issue_prefetch = [&](uint32_t c, int b) {
        if (tid == 0 && chunk_tma(c)) {
            const uint32_t mb = b ? mb1 : mb0;
            const uint32_t bytes = chunk_n(c) * 8;
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(bytes) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"((uint32_t)__cvta_generic_to_shared(st[b].words)), "l"(a.src + (uint64_t)c * kTaskWords),
                         "r"(bytes), "r"(mb) : "memory");
        }
        const uint64_t mw = (uint64_t)c * kMaskPerTask + tid;
        if (tid < kMaskPerTask) pf_mask = mw < n_mask ? a.mask[mw] : 0u;
        if (tid == kMaskPerTask) { pf_cb0 = a.chunk_base[c]; pf_cb1 = a.chunk_base[c + 1]; }
    };
    auto commit_prefetch = [&](int b) {
        if (tid < kMaskPerTask) st[b].mask[tid] = pf_mask;
        if (tid == kMaskPerTask) { st[b].rec0 = pf_cb0; st[b].nrec = pf_cb1 > pf_cb0 ? pf_cb1 - pf_cb0 : 0; }
    };

    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb0));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb1));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    uint32_t n_id = 0, n_rg = 0, n_st = 0;
    uint64_t first = ~0ull;
    uint32_t c = blockIdx.x;
    if (c < n_word_tasks) issue_prefetch(c, 0);
    for (uint32_t it = 0; c < n_word_tasks; ++it, c += word_ctas) {
        const int b = it & 1;
        Stage& S = st[b];
        const uint32_t n = chunk_n(c);
        const uint64_t ws = (uint64_t)c * kTaskWords;
        commit_prefetch(b);
        __syncthreads();  // stage b's mask / range visible; stage b^1 no longer read
        const uint32_t next = c + word_ctas;
        if (next < n_word_tasks) {
            if (tid == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // stage b^1's store has read its words
            issue_prefetch(next, b ^ 1);
        }
        if (!chunk_tma(c))
            for (uint32_t q = tid; q < n; q += kThreads) S.words[q] = ld_stream(a.src + ws + q);
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
        const uint64_t rec0 = S.rec0;
        const uint32_t n_rec = S.nrec;
        const uint32_t n_rec_c = min(n_rec, (uint32_t)kTaskWords);
        bool words_ready = !chunk_tma(c);
        for (uint32_t rb = 0; rb < max(n_rec_c, 1u); rb += 2 * kThreads) {
            uint64_t exp[2], nv[2];
            uint32_t kind[2];  // 0 ok, 1 bad id, 2 bad range, 3 none
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                const uint32_t r = rb + tid + u * kThreads;
                kind[u] = 3;
                exp[u] = nv[u] = 0;
                if (r < n_rec_c) {
                    kind[u] = 1;
                    const uint64_t k = rec0 + r;
                    if (k < a.n_slots) {
                        const uint64_t rec = a.slot[k];
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
            if (rb == 0) __syncthreads();  // prefix ready (and plain-loaded words)
            if (!words_ready) {
                mbar_wait(b ? mb1 : mb0, (it >> 1) & 1);
                words_ready = true;
            }
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                if (kind[u] == 3) continue;
                const uint32_t r = rb + tid + u * kThreads;
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
        if (tid == 0 && n_rec > (uint32_t)kTaskWords) n_id += n_rec - kTaskWords;
        __syncthreads();
        // the chunk's words back to HBM
        if (chunk_tma(c)) {
            if (tid == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                             ::"l"(a.dst + ws), "r"((uint32_t)__cvta_generic_to_shared(S.words)), "r"(n * 8) : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
        } else {
            for (uint32_t q = tid; q < n; q += kThreads) st_stream(a.dst + ws + q, S.words[q]);
        }
    }
    if (tid == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
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
    }
    const uint32_t n_word_tasks = (uint32_t)((a.n_words + kTaskWords - 1) / kTaskWords);
    const uint32_t n_node_tasks = a.func_id ? (a.n_nodes + kNodesPerTask - 1) / kNodesPerTask : 0;
    const uint32_t word_ctas = std::min<uint32_t>(n_word_tasks, (uint32_t)sm_count * 4);
    {
        TimedLaunch tl("restore_report_init", stream);
        report_init<<<1, 1, 0, stream>>>(a.report);
    }
    if (word_ctas + n_node_tasks) {
        TimedLaunch tl("restore", stream);
        restore_kernel<<<word_ctas + n_node_tasks, kThreads, 0, stream>>>(a, n_word_tasks, word_ctas, n_node_tasks);
    }
    return cudaGetLastError();
}

}  // namespace medusa
