// Shared device helpers and internal launch interfaces of libmedusa (sm_100a).
#pragma once
#include <cstdio>

#include <cstdint>
#include <utility>
#include <cuda_runtime.h>

#include "medusa.h"

namespace medusa {

constexpr uint32_t kChunkWords = MEDUSA_CHUNK_WORDS;
constexpr uint64_t kOffMask = (1ull << MEDUSA_OFF_BITS) - 1;

// ---- memory access helpers ---------------------------------------------------
// Streaming 16-byte access to the parameter image: no L1 allocation (every byte
// is touched exactly once).  Plain ld.global (not .nc) because restore may run
// in place.
__device__ __forceinline__ void ld_stream_v2(const uint64_t* p, uint64_t& a, uint64_t& b) {
    asm volatile("ld.global.L1::no_allocate.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p));
}
__device__ __forceinline__ void st_stream_v2(uint64_t* p, uint64_t a, uint64_t b) {
    asm volatile("st.global.L1::no_allocate.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ uint64_t ld_stream(const uint64_t* p) {
    uint64_t a;
    asm volatile("ld.global.L1::no_allocate.u64 %0, [%1];" : "=l"(a) : "l"(p));
    return a;
}
__device__ __forceinline__ void st_stream(uint64_t* p, uint64_t a) {
    asm volatile("st.global.L1::no_allocate.u64 [%0], %1;" ::"l"(p), "l"(a) : "memory");
}

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Position of the k-th (0-based) set bit of w; requires k < popc(w).  Five
// popcount halvings, branch-free (the __fns library sequence is ~3x as many
// instructions, with branches).
__device__ __forceinline__ uint32_t nth_set_bit(uint32_t w, uint32_t k) {
    uint32_t pos = 0, c;
    c = __popc(w & 0xFFFFu);
    if (k >= c) { k -= c; pos = 16; }
    c = __popc((w >> pos) & 0xFFu);
    if (k >= c) { k -= c; pos += 8; }
    c = __popc((w >> pos) & 0xFu);
    if (k >= c) { k -= c; pos += 4; }
    c = __popc((w >> pos) & 0x3u);
    if (k >= c) { k -= c; pos += 2; }
    c = (w >> pos) & 1u;
    return k >= c ? pos + 1 : pos;
}

// ---- programmatic dependent launch (PDL) --------------------------------------
// Kernels after the first of a call are launched with programmatic stream
// serialization: a grid may start while its predecessor drains.  Every kernel
// executes pdl_wait() (full completion + memory flush of the predecessor) before
// it touches anything the predecessor writes.  Most kernels call pdl_trigger()
// only after their own pdl_wait(), so "my predecessor has triggered" implies
// "everything before my predecessor is complete" and a kernel may read the
// outputs of kernels two or more launches back before it waits (k_buf_copy).  With MEDUSA_EARLY_TRIGGER the
// tail of a call -- k_emit, k_result, report_init -- triggers at its start, so
// each successor is resident and waiting when its predecessor completes; the
// restore then reads nothing a kernel of the stream wrote before its own
// pdl_wait() (the slot table and the kernel table after it; before it only its
// inputs: the image words and the kernel ids).  (ALL10 / C5 step -0.2 / -0.4
// us: measured, kept.)
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
#ifndef MEDUSA_EARLY_TRIGGER
#define MEDUSA_EARLY_TRIGGER 1
#endif
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), unsigned grid, unsigned block, size_t smem,
                              cudaStream_t stream, Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

// ---- instrumentation (api.cu) -------------------------------------------------
// Brackets one launch with events when the calling thread enabled timing.  While
// timing is on, materialize runs its branches serially on the caller's stream, so
// every kernel's duration is its own (no concurrent branch inside the events).
bool timing_enabled();
struct TimedLaunch {
    TimedLaunch(const char* name, cudaStream_t s);
    ~TimedLaunch();
    const char* name;
    cudaStream_t stream;
    void* slot;
};

// ---- timeline instrumentation (diagnostic builds only: -DMEDUSA_TIMELINE) ------
// Thread 0 of a CTA appends {start, end, kernel, cta, sm, tag} to a per-TU device
// buffer (tools/timeline.py builds libmedusa_tl.so and reads it back).
// ---- checked builds (-DMEDUSA_CHECKED; diagnostic, tools/gpu_variant_tests.sh) ----
// MCHECK(c): a device-side bounds / invariant check on the computed indices of
// the shared- and global-memory accesses that depend on data (positions from
// searches, counts, ranks); a failure traps the kernel, so the test that ran it
// fails with a CUDA error.  Compiled out of the product build.
#ifdef MEDUSA_CHECKED
#define MCHECK(c)                                                                          \
    do {                                                                                   \
        if (!(c)) {                                                                        \
            printf("MCHECK failed: %s at %s:%d (block %u thread %u)\n", #c, __FILE__, __LINE__, \
                   blockIdx.x, threadIdx.x);                                               \
            __trap();                                                                      \
        }                                                                                  \
    } while (0)
#else
#define MCHECK(c) ((void)0)
#endif

#ifdef MEDUSA_TIMELINE
struct TlRec {
    unsigned long long t0, t1;
    unsigned int kernel, cta, sm, tag;
};
__device__ __forceinline__ unsigned long long tl_now() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
#define MEDUSA_TL_DEFINE                                                                         \
    __device__ TlRec* g_tl = nullptr;                                                            \
    __device__ unsigned int g_tl_n = 0, g_tl_cap = 0;                                            \
    __device__ __forceinline__ void tl_rec(unsigned k, unsigned tag, unsigned long long t0) {    \
        if (threadIdx.x != 0 || !g_tl) return;                                                   \
        const unsigned i = atomicAdd(&g_tl_n, 1u);                                               \
        unsigned sm;                                                                             \
        asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));                                          \
        if (i < g_tl_cap) g_tl[i] = TlRec{t0, tl_now(), k, blockIdx.x, sm, tag};                 \
    }
#define TL_NOW() tl_now()
#define TL_REC(k, tag, t0) tl_rec((k), (tag), (t0))
#else
#pragma nv_diag_suppress 550  // timeline stamps are set but unused without MEDUSA_TIMELINE
#define MEDUSA_TL_DEFINE
#define TL_NOW() 0ull
#define TL_REC(k, tag, t0) ((void)(t0))
#endif
#define TL_PHASE(k, tag, var) \
    do {                      \
        TL_REC(k, tag, var);  \
        var = TL_NOW();       \
    } while (0)

// ---- restore (restore.cu) ------------------------------------------------------
struct RestoreArgs {
    const uint64_t* src;
    uint64_t* dst;
    uint64_t n_words;
    const uint32_t* mask;
    const uint32_t* chunk_base;
    const uint64_t* slot;
    uint64_t n_slots;  // records that may be read: min(n_slots, capacity)
    uint64_t slot_capacity;
    const uint64_t* old_base;
    const uint64_t* new_base;
    const uint64_t* new_size;
    uint32_t n_alloc;
    const uint32_t* func_id;
    uint64_t* func_out;
    uint32_t n_nodes;
    const uint64_t* table;
    uint32_t n_func;
    medusa_report* report;
};
cudaError_t launch_restore(const RestoreArgs& a, cudaStream_t stream);

// ---- materialize (materialize.cu) ---------------------------------------------
struct MaterializeArgs {
    const uint64_t* words;
    uint64_t n_words;
    const uint64_t* node_off;
    uint32_t n_nodes;
    const uint32_t* node_t;
    const medusa_alloc* alloc;
    uint32_t n_alloc;
    uint32_t* mask;
    uint32_t* chunk_base;
    uint64_t* slot;
    uint64_t capacity;
};
// Runs the whole analysis on `stream`, reads back the outcome and returns a
// status; *n_slots = slots found (0 on INVALID_ARG / TRACE).
medusa_status run_materialize(const MaterializeArgs& a, uint64_t* n_slots, cudaStream_t stream,
                              cudaError_t* cuda_err);
// Enqueues the analysis only; the outcome is written to *d_result.
medusa_status run_materialize_async(const MaterializeArgs& a, medusa_mat_result* d_result, cudaStream_t stream,
                                    cudaError_t* cuda_err);

// Live materialize scratch of the current device, in bytes; and its release
// (synchronizes the device, frees the scratch and every retired buffer).
uint64_t scratch_bytes();
cudaError_t release_scratch();

// ---- buffer contents (buffers.cu) ---------------------------------------------
medusa_status run_buffers_plan(const medusa_alloc* alloc, uint32_t n_alloc, const uint32_t* cap, uint32_t n_cap,
                               const uint64_t* slot, uint64_t n_slots, uint8_t* cls, uint32_t* perm,
                               uint64_t* perm_off, uint32_t capacity, uint32_t* h_n_perm, uint64_t* h_bytes,
                               cudaStream_t stream, cudaError_t* err);
cudaError_t launch_buffers_copy(bool to_blob, uint8_t* blob_w, const uint8_t* blob_r, const uint32_t* perm,
                                const uint64_t* perm_off, uint32_t n_perm, const uint64_t* base, const uint64_t* size,
                                uint32_t n_alloc, medusa_buf_report* rep, cudaStream_t stream);

}  // namespace medusa
