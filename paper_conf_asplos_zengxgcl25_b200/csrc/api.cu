// C-ABI entry points of libmedusa.so (include/medusa.h): argument checks,
// per-device kernel-address tables, status / error plumbing, instrumentation.
#include <algorithm>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace medusa {
namespace {

thread_local int g_last_cuda_error = 0;

medusa_status cuda_fail(cudaError_t e) {
    g_last_cuda_error = (int)e;
    return MEDUSA_ERR_CUDA;
}

// ---- per-device kernel address table (§5: filled from triggering kernels) ----
struct DeviceTable {
    uint64_t* d_table = nullptr;
    uint32_t capacity = 0;
    uint32_t n_func = 0;
    bool set = false;
    std::vector<uint64_t*> retired;  // earlier tables: a captured graph may still read them
};
std::mutex g_mu;
std::vector<DeviceTable> g_tables;

bool aligned8(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 7) == 0; }

// ---- instrumentation --------------------------------------------------------
struct TimingRec {
    const char* name;
    cudaEvent_t start, stop;
};
thread_local bool g_timing = false;
thread_local std::vector<TimingRec> g_timing_recs;
thread_local std::vector<cudaEvent_t> g_event_pool;  // events reused across reads (creating one per
                                                       // launch made the host slower than the GPU)

cudaEvent_t pooled_event() {
    if (!g_event_pool.empty()) {
        cudaEvent_t e = g_event_pool.back();
        g_event_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}

}  // namespace

bool timing_enabled() { return g_timing; }

TimedLaunch::TimedLaunch(const char* n, cudaStream_t s) : name(n), stream(s), slot(nullptr) {
    if (!g_timing) return;
    TimingRec r{n, pooled_event(), pooled_event()};
    cudaEventRecord(r.start, s);
    g_timing_recs.push_back(r);
    slot = reinterpret_cast<void*>(g_timing_recs.size());
}
TimedLaunch::~TimedLaunch() {
    if (!slot) return;
    cudaEventRecord(g_timing_recs[reinterpret_cast<size_t>(slot) - 1].stop, stream);
}

}  // namespace medusa

using namespace medusa;

extern "C" {

int medusa_last_cuda_error(void) { return g_last_cuda_error; }

const char* medusa_status_string(medusa_status s) {
    switch (s) {
        case MEDUSA_OK: return "MEDUSA_OK";
        case MEDUSA_ERR_INVALID_ARG: return "MEDUSA_ERR_INVALID_ARG";
        case MEDUSA_ERR_TRACE: return "MEDUSA_ERR_TRACE";
        case MEDUSA_ERR_CAPACITY: return "MEDUSA_ERR_CAPACITY";
        case MEDUSA_ERR_NO_TABLE: return "MEDUSA_ERR_NO_TABLE";
        case MEDUSA_ERR_CUDA: return "MEDUSA_ERR_CUDA";
        case MEDUSA_ERR_RETRY: return "MEDUSA_ERR_RETRY";
    }
    return "MEDUSA_UNKNOWN_STATUS";
}

void medusa_timing_enable(int on) { g_timing = on != 0; }

uint64_t medusa_scratch_bytes(void) { return scratch_bytes(); }

medusa_status medusa_scratch_release(void) {
    cudaError_t e = release_scratch();  // synchronizes the device
    if (e != cudaSuccess) return cuda_fail(e);
    int dev = 0;
    if ((e = cudaGetDevice(&dev)) != cudaSuccess) return cuda_fail(e);
    std::lock_guard<std::mutex> lk(g_mu);
    if ((int)g_tables.size() > dev) {
        for (uint64_t* p : g_tables[dev].retired) cudaFree(p);
        g_tables[dev].retired.clear();
    }
    return MEDUSA_OK;
}

int medusa_timing_read(const char** names, float* ms, int max) {
    int n = 0;
    for (auto& r : g_timing_recs) {
        if (n < max) {
            float t = 0.f;
            cudaEventSynchronize(r.stop);
            cudaEventElapsedTime(&t, r.start, r.stop);
            if (names) names[n] = r.name;
            if (ms) ms[n] = t;
            ++n;
        }
        g_event_pool.push_back(r.start);
        g_event_pool.push_back(r.stop);
    }
    g_timing_recs.clear();
    return n;
}

static medusa_status materialize_args(const uint64_t* d_words, uint64_t n_words, const uint64_t* d_node_word_off,
                                      uint32_t n_nodes, const uint32_t* d_node_t, const medusa_alloc* d_alloc,
                                      uint32_t n_alloc, const medusa_slots* slots) {
    if (!slots || !d_node_word_off || !slots->d_chunk_base) return MEDUSA_ERR_INVALID_ARG;
    if (n_words > 0 && (!d_words || !slots->d_mask)) return MEDUSA_ERR_INVALID_ARG;
    if (n_nodes > 0 && !d_node_t) return MEDUSA_ERR_INVALID_ARG;
    if (n_alloc > 0 && !d_alloc) return MEDUSA_ERR_INVALID_ARG;
    if (slots->capacity > 0 && !slots->d_slot) return MEDUSA_ERR_INVALID_ARG;
    if (n_alloc > (1u << MEDUSA_ID_BITS) || n_words > 0xFFFFFFFFull) return MEDUSA_ERR_INVALID_ARG;
    if (!aligned8(d_words) || !aligned8(d_node_word_off) || !aligned8(d_alloc) || !aligned8(slots->d_slot))
        return MEDUSA_ERR_INVALID_ARG;
    return MEDUSA_OK;
}

medusa_status medusa_materialize(const uint64_t* d_words, uint64_t n_words,
                                 const uint64_t* d_node_word_off, uint32_t n_nodes,
                                 const uint32_t* d_node_t, const medusa_alloc* d_alloc, uint32_t n_alloc,
                                 medusa_slots* slots, uint64_t* h_n_slots, cudaStream_t stream) {
    if (h_n_slots) *h_n_slots = 0;
    if (!h_n_slots) return MEDUSA_ERR_INVALID_ARG;
    medusa_status st = materialize_args(d_words, n_words, d_node_word_off, n_nodes, d_node_t, d_alloc, n_alloc, slots);
    if (st != MEDUSA_OK) return st;
    MaterializeArgs a{d_words, n_words, d_node_word_off, n_nodes, d_node_t, d_alloc, n_alloc,
                      slots->d_mask, slots->d_chunk_base, slots->d_slot, slots->capacity};
    cudaError_t ce = cudaSuccess;
    st = run_materialize(a, h_n_slots, stream, &ce);
    if (st == MEDUSA_ERR_CUDA) g_last_cuda_error = (int)ce;
    return st;
}

medusa_status medusa_materialize_async(const uint64_t* d_words, uint64_t n_words,
                                       const uint64_t* d_node_word_off, uint32_t n_nodes,
                                       const uint32_t* d_node_t, const medusa_alloc* d_alloc, uint32_t n_alloc,
                                       medusa_slots* slots, medusa_mat_result* d_result, cudaStream_t stream) {
    if (!d_result || !aligned8(d_result)) return MEDUSA_ERR_INVALID_ARG;
    medusa_status st = materialize_args(d_words, n_words, d_node_word_off, n_nodes, d_node_t, d_alloc, n_alloc, slots);
    if (st != MEDUSA_OK) return st;
    MaterializeArgs a{d_words, n_words, d_node_word_off, n_nodes, d_node_t, d_alloc, n_alloc,
                      slots->d_mask, slots->d_chunk_base, slots->d_slot, slots->capacity};
    cudaError_t ce = cudaSuccess;
    st = run_materialize_async(a, d_result, stream, &ce);
    if (st == MEDUSA_ERR_CUDA) g_last_cuda_error = (int)ce;
    return st;
}

#ifndef MEDUSA_TABLE_KERNEL
#define MEDUSA_TABLE_KERNEL 1
#endif
namespace medusa {
// the kernel-address table copy as a kernel: in a captured step a kernel node
// starts sooner than a copy-engine memcpy node, and the analysis that follows
// may start beside it (it triggers at once; the restore, two launches on, is
// the first kernel that reads the table)
static __global__ void k_table_copy(uint64_t* dst, const uint64_t* src, uint32_t n) {
    medusa::pdl_wait();  // the previous user of the table
    medusa::pdl_trigger();
    for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) dst[k] = src[k];
}
}  // namespace medusa

medusa_status medusa_kernel_table_set(const uint64_t* d_func_addr, uint32_t n_func, cudaStream_t stream) {
    if (n_func > 0 && (!d_func_addr || !aligned8(d_func_addr))) return MEDUSA_ERR_INVALID_ARG;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e);
    std::lock_guard<std::mutex> lk(g_mu);
    if ((int)g_tables.size() <= dev) g_tables.resize(dev + 1);
    DeviceTable& t = g_tables[dev];
    if (n_func > t.capacity) {
        uint32_t cap = n_func < 1024 ? 1024 : n_func;
        uint64_t* p = nullptr;
        e = cudaMalloc(&p, (size_t)cap * sizeof(uint64_t));
        if (e != cudaSuccess) return cuda_fail(e);
        // the old table stays allocated: restores in flight, and CUDA graphs that
        // captured a medusa_restore, hold its address (freed by medusa_scratch_release)
        if (t.d_table) t.retired.push_back(t.d_table);
        t.d_table = p;
        t.capacity = cap;
    }
    if (n_func > 0) {
        if (MEDUSA_TABLE_KERNEL) {
            medusa::TimedLaunch tl("table_copy", stream);
            e = medusa::launch_pdl(medusa::k_table_copy, std::min<uint32_t>((n_func + 255) / 256, 148u), 256, 0, stream, t.d_table,
                                   d_func_addr, n_func);
        } else {
            e = cudaMemcpyAsync(t.d_table, d_func_addr, (size_t)n_func * sizeof(uint64_t), cudaMemcpyDeviceToDevice,
                                stream);
        }
        if (e != cudaSuccess) return cuda_fail(e);
    }
    t.n_func = n_func;
    t.set = true;
    return MEDUSA_OK;
}

medusa_status medusa_restore(const uint64_t* d_src_words, uint64_t* d_dst_words, uint64_t n_words,
                             const medusa_slots* slots, uint64_t n_slots, const uint64_t* d_old_base,
                             const uint64_t* d_new_base, const uint64_t* d_new_size, uint32_t n_alloc,
                             const uint32_t* d_func_id, uint64_t* d_func_out, uint32_t n_nodes,
                             medusa_report* d_report, cudaStream_t stream) {
    if (!d_report || !slots || !aligned8(d_report)) return MEDUSA_ERR_INVALID_ARG;
    const bool from_table = n_slots == MEDUSA_N_SLOTS_FROM_TABLE;
    if (n_words > 0xFFFFFFFFull || (!from_table && n_slots > n_words)) return MEDUSA_ERR_INVALID_ARG;
    if (n_words > 0) {
        if (!d_src_words || !d_dst_words || !slots->d_mask || !slots->d_chunk_base) return MEDUSA_ERR_INVALID_ARG;
        if (!aligned8(d_src_words) || !aligned8(d_dst_words)) return MEDUSA_ERR_INVALID_ARG;
        const uintptr_t s = reinterpret_cast<uintptr_t>(d_src_words), d = reinterpret_cast<uintptr_t>(d_dst_words);
        const uintptr_t bytes = (uintptr_t)n_words * 8;
        if (s != d && s < d + bytes && d < s + bytes) return MEDUSA_ERR_INVALID_ARG;  // partial overlap
    }
    if (from_table) n_slots = slots->capacity;  // bound only: the table's chunk prefix gives the ranges
    if (n_slots > 0 && (!slots->d_slot || !aligned8(slots->d_slot))) return MEDUSA_ERR_INVALID_ARG;
    if (n_alloc > 0 && (!d_old_base || !d_new_base || !d_new_size)) return MEDUSA_ERR_INVALID_ARG;
    const bool gather = d_func_id || d_func_out || n_nodes;
    if (gather && (!d_func_id || !d_func_out || n_nodes == 0 || !aligned8(d_func_out))) return MEDUSA_ERR_INVALID_ARG;

    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e);
    const uint64_t* table = nullptr;
    uint32_t n_func = 0;
    if (gather) {
        std::lock_guard<std::mutex> lk(g_mu);
        if ((int)g_tables.size() <= dev || !g_tables[dev].set) return MEDUSA_ERR_NO_TABLE;
        table = g_tables[dev].d_table;
        n_func = g_tables[dev].n_func;
    }
    RestoreArgs a{d_src_words, d_dst_words, n_words, slots->d_mask, slots->d_chunk_base, slots->d_slot,
                  n_slots < slots->capacity ? n_slots : slots->capacity, slots->capacity, d_old_base, d_new_base, d_new_size,
                  n_alloc, gather ? d_func_id : nullptr, d_func_out, gather ? n_nodes : 0, table, n_func,
                  d_report};
    e = launch_restore(a, stream);
    if (e != cudaSuccess) return cuda_fail(e);
    return MEDUSA_OK;
}

medusa_status medusa_buffers_plan(const medusa_alloc* d_alloc, uint32_t n_alloc, const uint32_t* d_capture_t,
                                  uint32_t n_capture, const uint64_t* d_slot, uint64_t n_slots, uint8_t* d_class,
                                  uint32_t* d_perm, uint64_t* d_perm_off, uint32_t perm_capacity,
                                  uint32_t* h_n_perm, uint64_t* h_blob_bytes, cudaStream_t stream) {
    if (h_n_perm) *h_n_perm = 0;
    if (h_blob_bytes) *h_blob_bytes = 0;
    if (!h_n_perm || !h_blob_bytes || !d_perm_off || !aligned8(d_perm_off)) return MEDUSA_ERR_INVALID_ARG;
    if (n_alloc > 0 && (!d_alloc || !d_class || !aligned8(d_alloc))) return MEDUSA_ERR_INVALID_ARG;
    if (n_capture > 0 && (!d_capture_t || (reinterpret_cast<uintptr_t>(d_capture_t) & 3))) return MEDUSA_ERR_INVALID_ARG;
    if (n_slots > 0 && (!d_slot || !aligned8(d_slot))) return MEDUSA_ERR_INVALID_ARG;
    if (perm_capacity > 0 && (!d_perm || (reinterpret_cast<uintptr_t>(d_perm) & 3))) return MEDUSA_ERR_INVALID_ARG;
    cudaError_t ce = cudaSuccess;
    medusa_status st = run_buffers_plan(d_alloc, n_alloc, d_capture_t, n_capture, d_slot, n_slots, d_class, d_perm,
                                        d_perm_off, perm_capacity, h_n_perm, h_blob_bytes, stream, &ce);
    if (st == MEDUSA_ERR_CUDA) g_last_cuda_error = (int)ce;
    return st;
}

static medusa_status buffers_copy_args(const uint32_t* d_perm, const uint64_t* d_perm_off, uint32_t n_perm,
                                       const void* d_blob, medusa_buf_report* d_report) {
    if (!d_report || !aligned8(d_report) || !d_perm_off || !aligned8(d_perm_off)) return MEDUSA_ERR_INVALID_ARG;
    if (n_perm > 0 && (!d_perm || (reinterpret_cast<uintptr_t>(d_perm) & 3))) return MEDUSA_ERR_INVALID_ARG;
    if (n_perm > 0 && (!d_blob || (reinterpret_cast<uintptr_t>(d_blob) & 15))) return MEDUSA_ERR_INVALID_ARG;
    return MEDUSA_OK;
}

medusa_status medusa_buffers_save(const uint32_t* d_perm, const uint64_t* d_perm_off, uint32_t n_perm,
                                  const uint64_t* d_base, uint32_t n_alloc, uint8_t* d_blob,
                                  medusa_buf_report* d_report, cudaStream_t stream) {
    medusa_status st = buffers_copy_args(d_perm, d_perm_off, n_perm, d_blob, d_report);
    if (st != MEDUSA_OK) return st;
    if (n_alloc > 0 && (!d_base || !aligned8(d_base))) return MEDUSA_ERR_INVALID_ARG;
    cudaError_t e = launch_buffers_copy(true, d_blob, nullptr, d_perm, d_perm_off, n_perm, d_base, nullptr, n_alloc,
                                        d_report, stream);
    return e == cudaSuccess ? MEDUSA_OK : cuda_fail(e);
}

medusa_status medusa_buffers_restore(const uint8_t* d_blob, const uint32_t* d_perm, const uint64_t* d_perm_off,
                                     uint32_t n_perm, const uint64_t* d_new_base, const uint64_t* d_new_size,
                                     uint32_t n_alloc, medusa_buf_report* d_report, cudaStream_t stream) {
    medusa_status st = buffers_copy_args(d_perm, d_perm_off, n_perm, d_blob, d_report);
    if (st != MEDUSA_OK) return st;
    if (n_alloc > 0 && (!d_new_base || !d_new_size || !aligned8(d_new_base) || !aligned8(d_new_size)))
        return MEDUSA_ERR_INVALID_ARG;
    cudaError_t e = launch_buffers_copy(false, nullptr, d_blob, d_perm, d_perm_off, n_perm, d_new_base, d_new_size,
                                        n_alloc, d_report, stream);
    return e == cudaSuccess ? MEDUSA_OK : cuda_fail(e);
}

}  // extern "C"
