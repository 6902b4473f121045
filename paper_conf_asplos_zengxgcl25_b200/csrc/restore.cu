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
//   * one CTA of 128 threads per task of 1024 words (half a MEDUSA_CHUNK); a
//     thread moves four 16-byte pairs with streaming (L1::no_allocate) vector
//     loads issued up front, so ~16 KB per CTA is in flight;
//   * the task's slot records are contiguous ([chunk_base + popc prefix, ...)),
//     so they are fetched coalesced into shared memory and the three per-slot
//     base-table gathers (L2-resident: 24 B per allocation) are issued per
//     record, not per word; each word then finds its record by
//     popc(mask & lanemask) + a shared 32-entry exclusive scan;
//   * gather tasks (1024 nodes each) are appended to the same grid;
//   * validation failures are aggregated per CTA in shared memory and folded
//     into the report with one atomic per counter; the last CTA (ticket in
//     report->reserved) converts the min-trackers and clears the ticket.
#include "common.cuh"

namespace medusa {
namespace {

constexpr int kTaskWords = 1024;
constexpr int kThreads = 128;
constexpr int kPairsPerThread = kTaskWords / 2 / kThreads;  // 4
constexpr int kMaskPerTask = kTaskWords / 32;                // 32
constexpr int kNodesPerTask = 1024;

enum : uint8_t { REC_OK = 0, REC_BAD_ID = 1, REC_BAD_RANGE = 2 };

// report fields while in flight: counts accumulate; first_* hold the bitwise
// complement of the least index (0 = none) so that atomicMax tracks the min.
__device__ __forceinline__ void report_bad(unsigned long long* s_first, unsigned long long comp) {
    atomicMax(s_first, comp);  // comp = ~(least failing index seen by this thread)
}

__global__ void __launch_bounds__(kThreads)
restore_kernel(RestoreArgs a, uint32_t n_word_tasks, uint32_t n_tasks) {
    __shared__ uint32_t s_mask[kMaskPerTask];
    __shared__ uint32_t s_pre[kMaskPerTask + 1];
    __shared__ uint64_t s_expect[kTaskWords];
    __shared__ uint64_t s_newv[kTaskWords];
    __shared__ uint8_t s_kind[kTaskWords];
    __shared__ unsigned long long s_cnt[4];  // bad id, bad range, stale, bad func
    __shared__ unsigned long long s_first_word, s_first_node;
    __shared__ uint32_t s_base_rec, s_prev_pop;

    const int tid = threadIdx.x;
    const uint32_t task = blockIdx.x;
    if (tid < 4) s_cnt[tid] = 0;
    if (tid == 0) { s_first_word = 0; s_first_node = 0; s_prev_pop = 0; }

    if (task < n_word_tasks) {
        const uint64_t ws = (uint64_t)task * kTaskWords;
        const uint64_t we = min(ws + kTaskWords, a.n_words);
        // 1. issue the streaming loads of this task's words first
        uint64_t v[2 * kPairsPerThread];
        const bool vec = ((reinterpret_cast<uintptr_t>(a.src) | reinterpret_cast<uintptr_t>(a.dst)) & 15) == 0;
#pragma unroll
        for (int k = 0; k < kPairsPerThread; ++k) {
            const uint64_t g = ws + 2ull * (tid + k * kThreads);
            if (vec && g + 1 < we) {
                ld_stream_v2(a.src + g, v[2 * k], v[2 * k + 1]);
            } else {
                v[2 * k] = g < we ? ld_stream(a.src + g) : 0;
                v[2 * k + 1] = g + 1 < we ? ld_stream(a.src + g + 1) : 0;
            }
        }
        // 2. mask words of the task, chunk prefix, and (second half of a chunk)
        //    the popcount of the chunk's first half
        const uint64_t n_mask = (a.n_words + 31) / 32;
        const uint64_t mw0 = ws / 32;
        const bool second_half = (ws % kChunkWords) != 0;
        if (tid < kMaskPerTask) {
            s_mask[tid] = (mw0 + tid < n_mask) ? a.mask[mw0 + tid] : 0u;
        } else if (tid < 2 * kMaskPerTask) {
            uint32_t pop = 0;
            if (second_half) pop = __popc(a.mask[mw0 - kMaskPerTask + (tid - kMaskPerTask)]);
            pop = __reduce_add_sync(0xffffffffu, pop);
            if (tid == kMaskPerTask) s_prev_pop = pop;
        } else if (tid == 2 * kMaskPerTask) {
            s_base_rec = a.chunk_base[ws / kChunkWords];
        }
        __syncthreads();
        if (tid < 32) {
            const uint32_t pop = __popc(s_mask[tid]);
            uint32_t incl = pop;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (tid >= d) incl += y;
            }
            s_pre[tid] = incl - pop;
            if (tid == 31) s_pre[32] = incl;
        }
        __syncthreads();
        // 3. this task's records: contiguous, fetched coalesced; per record the
        //    base-table gathers and the record-level checks
        const uint64_t rec0 = (uint64_t)s_base_rec + s_prev_pop;
        const uint32_t n_rec = s_pre[32];
        for (uint32_t r = tid; r < n_rec; r += kThreads) {
            const uint64_t k = rec0 + r;
            uint8_t kind = REC_BAD_ID;
            uint64_t exp = 0, nv = 0;
            if (k < a.n_slots) {
                const uint64_t rec = a.slot[k];
                const uint64_t id = rec >> MEDUSA_OFF_BITS;
                const uint64_t off = rec & kOffMask;
                if (id < a.n_alloc) {
                    const uint64_t sz = __ldg(a.new_size + id);
                    const uint64_t ob = __ldg(a.old_base + id);
                    const uint64_t nb = __ldg(a.new_base + id);
                    if (off < sz) {
                        kind = REC_OK;
                        exp = ob + off;
                        nv = nb + off;
                    } else {
                        kind = REC_BAD_RANGE;
                    }
                }
            }
            s_kind[r] = kind;
            s_expect[r] = exp;
            s_newv[r] = nv;
        }
        __syncthreads();
        // 4. rewrite slot words, validate, store
        uint32_t n_id = 0, n_rg = 0, n_st = 0;
        unsigned long long first = 0;
#pragma unroll
        for (int k = 0; k < kPairsPerThread; ++k) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const uint32_t q = 2 * (tid + k * kThreads) + h;  // word within task
                const uint32_t mw = s_mask[q >> 5];
                if ((mw >> (q & 31)) & 1u) {
                    const uint32_t r = s_pre[q >> 5] + __popc(mw & ((1u << (q & 31)) - 1u));
                    const uint8_t kind = s_kind[r];
                    const uint64_t g = ws + q;
                    bool bad = true;
                    if (kind == REC_OK) {
                        if (v[2 * k + h] == s_expect[r]) { v[2 * k + h] = s_newv[r]; bad = false; }
                        else ++n_st;
                    } else if (kind == REC_BAD_ID) {
                        ++n_id;
                    } else {
                        ++n_rg;
                    }
                    if (bad && ~g > first) first = ~g;
                }
            }
        }
#pragma unroll
        for (int k = 0; k < kPairsPerThread; ++k) {
            const uint64_t g = ws + 2ull * (tid + k * kThreads);
            if (vec && g + 1 < we) {
                st_stream_v2(a.dst + g, v[2 * k], v[2 * k + 1]);
            } else {
                if (g < we) st_stream(a.dst + g, v[2 * k]);
                if (g + 1 < we) st_stream(a.dst + g + 1, v[2 * k + 1]);
            }
        }
        if (n_id | n_rg | n_st) {
            if (n_id) atomicAdd(&s_cnt[0], (unsigned long long)n_id);
            if (n_rg) atomicAdd(&s_cnt[1], (unsigned long long)n_rg);
            if (n_st) atomicAdd(&s_cnt[2], (unsigned long long)n_st);
            report_bad(&s_first_word, first);
        }
    } else if (task < n_tasks) {
        const uint64_t j0 = (uint64_t)(task - n_word_tasks) * kNodesPerTask;
        uint32_t n_bad = 0;
        unsigned long long first = 0;
        for (int k = 0; k < kNodesPerTask / kThreads; ++k) {
            const uint64_t j = j0 + tid + k * kThreads;
            if (j < a.n_nodes) {
                const uint32_t f = a.func_id[j];
                uint64_t addr = 0;
                if (f < a.n_func) addr = __ldg(a.table + f);
                if (addr == 0) {
                    ++n_bad;
                    if (~j > first) first = ~j;
                }
                a.func_out[j] = addr;
            }
        }
        if (n_bad) {
            atomicAdd(&s_cnt[3], (unsigned long long)n_bad);
            report_bad(&s_first_node, first);
        }
    }
    __syncthreads();
    // fold this CTA into the report; the last CTA finalizes it
    if (tid == 0) {
        unsigned long long* rep = reinterpret_cast<unsigned long long*>(a.report);
        const unsigned long long bad_slots = s_cnt[0] + s_cnt[1] + s_cnt[2];
        if (bad_slots) {
            atomicAdd(rep + 0, bad_slots);
            atomicMax(rep + 1, s_first_word);
            if (s_cnt[0]) atomicAdd(rep + 2, s_cnt[0]);
            if (s_cnt[1]) atomicAdd(rep + 3, s_cnt[1]);
            if (s_cnt[2]) atomicAdd(rep + 4, s_cnt[2]);
        }
        if (s_cnt[3]) {
            atomicAdd(rep + 5, s_cnt[3]);
            atomicMax(rep + 6, s_first_node);
        }
        __threadfence();
        const unsigned long long ticket = atomicAdd(rep + 7, 1ull);
        if (ticket == gridDim.x - 1) {
            __threadfence();
            rep[1] = ~atomicAdd(rep + 1, 0ull);
            rep[6] = ~atomicAdd(rep + 6, 0ull);
            rep[7] = 0;
        }
    }
}

}  // namespace

cudaError_t launch_restore(const RestoreArgs& a, cudaStream_t stream) {
    const uint32_t n_word_tasks = (uint32_t)((a.n_words + kTaskWords - 1) / kTaskWords);
    const uint32_t n_node_tasks = a.func_id ? (a.n_nodes + kNodesPerTask - 1) / kNodesPerTask : 0;
    const uint32_t n_tasks = n_word_tasks + n_node_tasks;
    cudaError_t e = cudaMemsetAsync(a.report, 0, sizeof(medusa_report), stream);
    if (e != cudaSuccess) return e;
    {
        TimedLaunch tl("restore", stream);
        restore_kernel<<<n_tasks ? n_tasks : 1, kThreads, 0, stream>>>(a, n_word_tasks, n_tasks);
    }
    return cudaGetLastError();
}

}  // namespace medusa
