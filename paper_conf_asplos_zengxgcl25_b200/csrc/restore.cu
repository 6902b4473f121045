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
//   * one CTA of 256 threads per 2048-word chunk; a thread moves four 16-byte
//     pairs with streaming (L1::no_allocate) vector loads issued first, so
//     32 KB per CTA is in flight;
//   * the chunk's records are the contiguous range [chunk_base[c],
//     chunk_base[c+1]), known after one load -- fetched coalesced into shared
//     memory with the three base-table gathers (L2-resident: 24 B per
//     allocation) done per record, not per word, while the mask's prefix
//     popcounts are scanned; a word finds its record at
//     prefix[mask word] + popc(mask & lanemask);
//   * gather tasks (2048 nodes each) are appended to the same grid;
//   * validation failures (rare) go to the report with atomics; a one-thread
//     kernel initializes the report first, so CTAs need no fence or ticket.
#include "common.cuh"

namespace medusa {
namespace {

constexpr int kTaskWords = MEDUSA_CHUNK_WORDS;  // 2048
constexpr int kThreads = 256;
constexpr int kPairsPerThread = kTaskWords / 2 / kThreads;  // 4
constexpr int kMaskPerTask = kTaskWords / 32;                // 64
constexpr int kNodesPerTask = 2048;

enum : uint8_t { REC_OK = 0, REC_BAD_ID = 1, REC_BAD_RANGE = 2 };

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

__global__ void __launch_bounds__(kThreads)
restore_kernel(RestoreArgs a, uint32_t n_word_tasks, uint32_t n_tasks) {
    __shared__ uint32_t s_mask[kMaskPerTask];
    __shared__ uint32_t s_pre[kMaskPerTask];
    __shared__ uint64_t s_expect[kTaskWords];
    __shared__ uint64_t s_newv[kTaskWords];
    __shared__ uint8_t s_kind[kTaskWords];
    __shared__ uint32_t s_rec0, s_nrec;

    const int tid = threadIdx.x;
    const uint32_t task = blockIdx.x;
    unsigned long long* rep = reinterpret_cast<unsigned long long*>(a.report);

    if (task < n_word_tasks) {
        const uint64_t ws = (uint64_t)task * kTaskWords;
        const uint64_t we = min(ws + kTaskWords, a.n_words);
        // 1. the words first (streaming, 16 B per load), then mask and record range
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
        const uint64_t n_mask = (a.n_words + 31) / 32;
        const uint64_t mw0 = ws / 32;
        if (tid < kMaskPerTask) {
            s_mask[tid] = (mw0 + tid < n_mask) ? a.mask[mw0 + tid] : 0u;
        } else if (tid == kMaskPerTask) {
            const uint32_t r0 = a.chunk_base[task], r1 = a.chunk_base[task + 1];
            s_rec0 = r0;
            s_nrec = r1 > r0 ? r1 - r0 : 0;
        }
        __syncthreads();
        // 2. warp 0: exclusive scan of the 64 mask popcounts; everyone: records
        if (tid < 32) {
            const uint32_t p0 = __popc(s_mask[2 * tid]), p1 = __popc(s_mask[2 * tid + 1]);
            uint32_t incl = p0 + p1;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (tid >= d) incl += y;
            }
            s_pre[2 * tid] = incl - p0 - p1;
            s_pre[2 * tid + 1] = incl - p1;
        }
        const uint64_t rec0 = s_rec0;
        const uint32_t n_rec = min(s_nrec, (uint32_t)kTaskWords);
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
        // 3. rewrite slot words, validate, store
        uint32_t n_id = 0, n_rg = 0, n_st = 0;
        uint64_t first = ~0ull;
#pragma unroll
        for (int k = 0; k < kPairsPerThread; ++k) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const uint32_t q = 2 * (tid + k * kThreads) + h;  // word within the chunk
                const uint32_t mw = s_mask[q >> 5];
                if ((mw >> (q & 31)) & 1u) {
                    const uint32_t r = s_pre[q >> 5] + __popc(mw & ((1u << (q & 31)) - 1u));
                    bool bad = true;
                    if (r < n_rec) {
                        const uint8_t kind = s_kind[r];
                        if (kind == REC_OK) {
                            if (v[2 * k + h] == s_expect[r]) { v[2 * k + h] = s_newv[r]; bad = false; }
                            else ++n_st;
                        } else if (kind == REC_BAD_ID) {
                            ++n_id;
                        } else {
                            ++n_rg;
                        }
                    } else {
                        ++n_id;  // table shorter than its mask says: no record to apply
                    }
                    if (bad) first = min(first, ws + q);
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
            atomicAdd(rep + 0, (unsigned long long)(n_id + n_rg + n_st));
            atomicMin(rep + 1, (unsigned long long)first);
            if (n_id) atomicAdd(rep + 2, (unsigned long long)n_id);
            if (n_rg) atomicAdd(rep + 3, (unsigned long long)n_rg);
            if (n_st) atomicAdd(rep + 4, (unsigned long long)n_st);
        }
    } else if (task < n_tasks) {
        const uint64_t j0 = (uint64_t)(task - n_word_tasks) * kNodesPerTask;
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
    }
}

}  // namespace

cudaError_t launch_restore(const RestoreArgs& a, cudaStream_t stream) {
    const uint32_t n_word_tasks = (uint32_t)((a.n_words + kTaskWords - 1) / kTaskWords);
    const uint32_t n_node_tasks = a.func_id ? (a.n_nodes + kNodesPerTask - 1) / kNodesPerTask : 0;
    const uint32_t n_tasks = n_word_tasks + n_node_tasks;
    {
        TimedLaunch tl("restore_report_init", stream);
        report_init<<<1, 1, 0, stream>>>(a.report);
    }
    if (n_tasks) {
        TimedLaunch tl("restore", stream);
        restore_kernel<<<n_tasks, kThreads, 0, stream>>>(a, n_word_tasks, n_tasks);
    }
    return cudaGetLastError();
}

}  // namespace medusa
