// Tracing device allocator for real-capture workloads.
// Not part of libmedusa: it produces the allocation trace that medusa_materialize
// consumes, from a real PyTorch model captured into a CUDA graph.
//
// Plugged into PyTorch as a CUDAPluggableAllocator behind a torch.cuda.MemPool,
// it serves the pool's segment requests (PyTorch's caching allocator still
// carves tensors out of them) from one of two pre-reserved arenas, and logs every
// allocation and free in call order with the number of nodes the capturing
// graph held at that moment -- which places each allocation event exactly
// between two kernel launches (one total order of allocations and
// launches).  Arena 1 plays the "online" process: its addresses differ, and
// replaying the same request sequence there yields the new bases.
#include <cuda_runtime.h>

#include <sys/types.h>

#include <cstdint>
#include <map>
#include <mutex>
#include <vector>

namespace {

struct Event {
    int64_t kind;         // 1 alloc, 2 free, 3 / 4 capture begin / end
    uint64_t ptr, size;
    int64_t nodes;        // nodes in the capturing graph at the call; -1 if not capturing
    int64_t capture;      // capture sequence number (ta_capture_begin), -1 if not capturing
};

struct Arena {
    char* base = nullptr;
    uint64_t size = 0;
    std::map<uint64_t, uint64_t> free_blocks;  // address -> size (coalesced)
    std::map<uint64_t, uint64_t> used;         // address -> size
};

std::mutex g_mu;
Arena g_arena[2];
int g_active = 0;
bool g_log = false;
int64_t g_capture = -1;
std::vector<Event> g_events;

constexpr uint64_t kAlign = 512;

void* arena_alloc(Arena& a, uint64_t size) {
    size = (size + kAlign - 1) / kAlign * kAlign;
    if (size == 0) size = kAlign;
    // best fit, lowest address among equals (deterministic)
    auto best = a.free_blocks.end();
    for (auto it = a.free_blocks.begin(); it != a.free_blocks.end(); ++it)
        if (it->second >= size && (best == a.free_blocks.end() || it->second < best->second)) best = it;
    if (best == a.free_blocks.end()) return nullptr;
    const uint64_t addr = best->first, bsz = best->second;
    a.free_blocks.erase(best);
    if (bsz > size) a.free_blocks[addr + size] = bsz - size;
    a.used[addr] = size;
    return reinterpret_cast<void*>(addr);
}

void arena_free(Arena& a, uint64_t addr) {
    auto it = a.used.find(addr);
    if (it == a.used.end()) return;
    uint64_t size = it->second;
    a.used.erase(it);
    auto nx = a.free_blocks.lower_bound(addr);
    if (nx != a.free_blocks.end() && addr + size == nx->first) { size += nx->second; a.free_blocks.erase(nx); }
    auto pv = a.free_blocks.lower_bound(addr);
    if (pv != a.free_blocks.begin()) {
        --pv;
        if (pv->first + pv->second == addr) { addr = pv->first; size += pv->second; a.free_blocks.erase(pv); }
    }
    a.free_blocks[addr] = size;
}

int64_t captured_nodes(cudaStream_t stream) {
    cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
    cudaGraph_t graph = nullptr;
    unsigned long long id = 0;
    if (cudaStreamGetCaptureInfo(stream, &st, &id, &graph, nullptr, nullptr) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    if (st != cudaStreamCaptureStatusActive || !graph) return -1;
    size_t n = 0;
    if (cudaGraphGetNodes(graph, nullptr, &n) != cudaSuccess) { cudaGetLastError(); return -1; }
    return (int64_t)n;
}

}  // namespace

extern "C" {

// Reserve the two arenas (bytes each) on the current device.  0 on success.
int ta_init(uint64_t bytes) {
    std::lock_guard<std::mutex> lk(g_mu);
    for (int k = 0; k < 2; ++k) {
        if (g_arena[k].base) continue;
        void* p = nullptr;
        if (cudaMalloc(&p, bytes) != cudaSuccess) return -1;
        g_arena[k].base = static_cast<char*>(p);
        g_arena[k].size = bytes;
        g_arena[k].free_blocks.clear();
        g_arena[k].used.clear();
        g_arena[k].free_blocks[reinterpret_cast<uint64_t>(p)] = bytes;
    }
    return 0;
}

// Which arena serves requests (0 = materialization-time process, 1 = online process).
void ta_select(int which) { std::lock_guard<std::mutex> lk(g_mu); g_active = which ? 1 : 0; }
void ta_log(int on) { std::lock_guard<std::mutex> lk(g_mu); g_log = on != 0; }
// capture markers (kind 3 = begin, 4 = end of capture `seq`) in the event log
void ta_capture_begin(int64_t seq) {
    std::lock_guard<std::mutex> lk(g_mu);
    g_capture = seq;
    if (g_log) g_events.push_back(Event{3, 0, 0, -1, seq});
}
void ta_capture_end() {
    std::lock_guard<std::mutex> lk(g_mu);
    if (g_log) g_events.push_back(Event{4, 0, 0, -1, g_capture});
    g_capture = -1;
}

// The CUDAPluggableAllocator entry points.
void* ta_malloc(ssize_t size, int device, cudaStream_t stream) {
    (void)device;
    const int64_t nodes = captured_nodes(stream);
    std::lock_guard<std::mutex> lk(g_mu);
    void* p = arena_alloc(g_arena[g_active], (uint64_t)size);
    if (p && g_log) g_events.push_back(Event{1, reinterpret_cast<uint64_t>(p), (uint64_t)size, nodes, nodes >= 0 ? g_capture : -1});
    return p;
}

void ta_free(void* ptr, ssize_t size, int device, cudaStream_t stream) {
    (void)device;
    const int64_t nodes = captured_nodes(stream);
    std::lock_guard<std::mutex> lk(g_mu);
    if (g_log) g_events.push_back(Event{2, reinterpret_cast<uint64_t>(ptr), (uint64_t)size, nodes, nodes >= 0 ? g_capture : -1});
    for (auto& a : g_arena)
        if (a.used.count(reinterpret_cast<uint64_t>(ptr))) arena_free(a, reinterpret_cast<uint64_t>(ptr));
}

// Replay helper for the online process: allocate without logging into the active arena.
uint64_t ta_raw_malloc(uint64_t size) {
    std::lock_guard<std::mutex> lk(g_mu);
    return reinterpret_cast<uint64_t>(arena_alloc(g_arena[g_active], size));
}

// Copy out up to `max` events as 5 int64 each; returns the number logged.
int64_t ta_events(int64_t* out, int64_t max) {
    std::lock_guard<std::mutex> lk(g_mu);
    const int64_t n = (int64_t)g_events.size();
    for (int64_t i = 0; i < n && i < max; ++i) {
        out[5 * i + 0] = g_events[i].kind;
        out[5 * i + 1] = (int64_t)g_events[i].ptr;
        out[5 * i + 2] = (int64_t)g_events[i].size;
        out[5 * i + 3] = g_events[i].nodes;
        out[5 * i + 4] = g_events[i].capture;
    }
    return n;
}

void ta_clear() { std::lock_guard<std::mutex> lk(g_mu); g_events.clear(); }

uint64_t ta_arena_base(int which) { return reinterpret_cast<uint64_t>(g_arena[which ? 1 : 0].base); }

}  // extern "C"
