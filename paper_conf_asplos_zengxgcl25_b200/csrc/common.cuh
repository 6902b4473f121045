// Shared device helpers and internal launch interfaces of libmedusa (sm_100a).
#pragma once

#include <cstdint>
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

// ---- instrumentation (api.cu) -------------------------------------------------
// Brackets one launch with events when the calling thread enabled timing.
struct TimedLaunch {
    TimedLaunch(const char* name, cudaStream_t s);
    ~TimedLaunch();
    const char* name;
    cudaStream_t stream;
    void* slot;
};

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

}  // namespace medusa
