// Copy-free buffer contents restoration (§4.3).
//
// Of the buffers the graph nodes' parameters point to, only the
// permanent ones need their contents saved offline and restored online:
// model-parameter buffers are "allocated before the CUDA graphs capturing"
// and hold the weights the serving process loads anyway; temporary
// buffers are allocated during a capture and "deallocated after capturing"
// (P:222), their contents are produced by the graph itself.  What remains --
// allocated during a capture and never freed -- is saved (two 4-byte
// buffers for 9.0% of the kernels).  DESIGN.md readings R-B1..R-B4.
//
// medusa_buffers_plan (offline, synchronous):
//   memset(class) -> k_buf_mark (one flag per allocation a slot refers to)
//   -> k_buf_class (tile of 1024 allocations per CTA: capture-interval search,
//      class, per-tile PERM count and bytes) -> k_buf_scatter (tile prefix by
//      one CTA-wide reduction over the per-tile counts, CTA scan, PERM ordinals
//      and blob offsets in ordinal order).
// medusa_buffers_save / medusa_buffers_restore (asynchronous, capturable):
//   k_buf_init (report) -> k_buf_copy (PDL): warps walk the blob in 2 KB
//   tasks; the segment holding a task's first byte comes from a warp-
//   cooperative 32-ary search over the segment offsets (ballot + clz, three
//   rounds for 24k segments); the warp then loads the descriptors of the next
//   32 segments at once (one lane each) into shared memory, and each lane
//   moves its four 16-byte units with vector loads issued before the stores
//   (byte loop where a unit straddles segments or the target address is not
//   16-byte aligned).  Both sides are contiguous runs, so the copy is
//   coalesced; the pass is HBM-bound at 2 bytes moved per blob byte.
#include <algorithm>

#include "common.cuh"

namespace medusa {
namespace {

constexpr int kPlanThreads = 256;
constexpr int kPlanPer = 4;
constexpr int kTile = kPlanThreads * kPlanPer;  // allocations per plan CTA
constexpr int kCopyThreads = 256;
constexpr uint32_t kTaskBytes = 1024;  // blob bytes per warp task (32 lanes x 2 units x 16 B)

struct PlanResult {
    uint32_t bad_capture;
    uint32_t pad;
    uint64_t n_perm;
    uint64_t bytes;
};

__global__ void k_buf_mark(const uint64_t* __restrict__ slot, uint64_t n_slots, uint32_t n_alloc,
                           uint8_t* __restrict__ cls) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n_slots; k += stride) {
        const uint64_t id = __ldg(slot + k) >> MEDUSA_OFF_BITS;
        if (id < n_alloc) cls[id] = 1;  // referenced by a node parameter; idempotent
    }
}

// Block-wide inclusive scan of (count, bytes) pairs; returns the exclusive
// prefix of this thread and the block totals.
__device__ __forceinline__ void block_scan2(uint32_t c, uint64_t b, uint32_t& c_ex, uint64_t& b_ex, uint32_t& c_tot,
                                            uint64_t& b_tot) {
    __shared__ uint32_t s_c[kPlanThreads / 32];
    __shared__ uint64_t s_b[kPlanThreads / 32];
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t ci = c;
    uint64_t bi = b;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t yc = __shfl_up_sync(0xffffffffu, ci, d);
        const uint64_t yb = __shfl_up_sync(0xffffffffu, bi, d);
        if (lane >= (uint32_t)d) { ci += yc; bi += yb; }
    }
    if (lane == 31) { s_c[warp] = ci; s_b[warp] = bi; }
    __syncthreads();
    uint32_t wc = 0, tc = 0;
    uint64_t wb = 0, tb = 0;
#pragma unroll
    for (int w = 0; w < kPlanThreads / 32; ++w) {
        if ((uint32_t)w < warp) { wc += s_c[w]; wb += s_b[w]; }
        tc += s_c[w];
        tb += s_b[w];
    }
    c_ex = wc + ci - c;
    b_ex = wb + bi - b;
    c_tot = tc;
    b_tot = tb;
    __syncthreads();
}

__global__ void __launch_bounds__(kPlanThreads)
k_buf_class(const medusa_alloc* __restrict__ alloc, uint32_t n_alloc, const uint32_t* __restrict__ cap,
            uint32_t n_cap, uint8_t* __restrict__ cls, uint32_t* __restrict__ tile_cnt,
            uint64_t* __restrict__ tile_bytes, PlanResult* res) {
    // capture intervals: begin < end, sorted, disjoint (graphs are captured one
    // at a time); checked by CTA 0
    if (blockIdx.x == 0) {
        for (uint32_t k = threadIdx.x; k < n_cap; k += kPlanThreads) {
            const uint32_t b = cap[2 * k], e = cap[2 * k + 1];
            if (!(b < e) || (k + 1 < n_cap && !(e <= cap[2 * k + 2]))) atomicOr(&res->bad_capture, 1u);
        }
    }
    const uint64_t i0 = (uint64_t)blockIdx.x * kTile + (uint64_t)threadIdx.x * kPlanPer;
    uint32_t cnt = 0;
    uint64_t bytes = 0;
#pragma unroll
    for (int q = 0; q < kPlanPer; ++q) {
        const uint64_t i = i0 + q;
        if (i >= n_alloc || cls[i] == 0) continue;
        const uint32_t ta = alloc[i].t_alloc, tf = alloc[i].t_free;
        // the capture with the greatest begin below t_alloc is the only one that
        // can contain it
        uint32_t lo = 0, hi = n_cap;  // count of begins < ta
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (__ldg(cap + 2 * mid) < ta) lo = mid + 1; else hi = mid;
        }
        const bool during = lo > 0 && ta < __ldg(cap + 2 * (lo - 1) + 1);
        uint8_t c;
        if (!during) c = MEDUSA_BUF_PARAM;             // allocated before capturing
        else if (tf != MEDUSA_T_END) c = MEDUSA_BUF_TEMP;  // deallocated after capturing
        else c = MEDUSA_BUF_PERM;                      // used across graph launches
        cls[i] = c;
        if (c == MEDUSA_BUF_PERM) {
            ++cnt;
            bytes += alloc[i].size;
        }
    }
    uint32_t c_ex, c_tot;
    uint64_t b_ex, b_tot;
    block_scan2(cnt, bytes, c_ex, b_ex, c_tot, b_tot);
    if (threadIdx.x == 0) {
        tile_cnt[blockIdx.x] = c_tot;
        tile_bytes[blockIdx.x] = b_tot;
    }
}

__global__ void __launch_bounds__(kPlanThreads)
k_buf_scatter(const medusa_alloc* __restrict__ alloc, uint32_t n_alloc, const uint8_t* __restrict__ cls,
              const uint32_t* __restrict__ tile_cnt, const uint64_t* __restrict__ tile_bytes, uint32_t n_tiles,
              uint32_t* __restrict__ perm, uint64_t* __restrict__ perm_off, uint32_t capacity, PlanResult* res) {
    // prefix of the tiles before this one: one CTA-wide reduction
    uint32_t pc = 0, ac = 0;
    uint64_t pb = 0, ab = 0;
    for (uint32_t t = threadIdx.x; t < n_tiles; t += kPlanThreads) {
        const uint32_t c = tile_cnt[t];
        const uint64_t b = tile_bytes[t];
        if (t < blockIdx.x) { pc += c; pb += b; }
        ac += c;
        ab += b;
    }
    uint32_t d0, d1;
    uint64_t e0, e1;
    block_scan2(pc, pb, d0, e0, pc, pb);
    block_scan2(ac, ab, d1, e1, ac, ab);
    const uint64_t i0 = (uint64_t)blockIdx.x * kTile + (uint64_t)threadIdx.x * kPlanPer;
    bool is_p[kPlanPer];
    uint64_t sz[kPlanPer];
    uint32_t cnt = 0;
    uint64_t bytes = 0;
#pragma unroll
    for (int q = 0; q < kPlanPer; ++q) {
        const uint64_t i = i0 + q;
        is_p[q] = i < n_alloc && cls[i] == MEDUSA_BUF_PERM;
        sz[q] = is_p[q] ? alloc[i].size : 0;
        cnt += is_p[q];
        bytes += sz[q];
    }
    uint32_t c_ex, c_tot;
    uint64_t b_ex, b_tot;
    block_scan2(cnt, bytes, c_ex, b_ex, c_tot, b_tot);
    uint64_t pos = (uint64_t)pc + c_ex, off = pb + b_ex;
#pragma unroll
    for (int q = 0; q < kPlanPer; ++q) {
        if (!is_p[q]) continue;
        if (pos < capacity) {
            perm[pos] = (uint32_t)(i0 + q);
            perm_off[pos] = off;
        }
        ++pos;
        off += sz[q];
    }
    if (blockIdx.x == n_tiles - 1 && threadIdx.x == 0) {
        if (ac <= capacity) perm_off[ac] = ab;
        res->n_perm = ac;
        res->bytes = ab;
    }
}

// Last k in [lo, hi) with off[k] <= p (off[lo] <= p assumed), found by the
// whole warp: 32 probes per round, ballot of the monotone predicate.
__device__ __forceinline__ uint32_t warp_last_le(const uint64_t* __restrict__ off, uint32_t lo, uint32_t hi,
                                                 uint64_t p) {
    const uint32_t lane = threadIdx.x & 31;
    while (hi - lo > 1) {
        const uint32_t stride = (hi - lo + 31) / 32;
        const uint32_t k = lo + lane * stride;
        const bool ok = k < hi && __ldg(off + k) <= p;
        const uint32_t m = 31 - __clz(__ballot_sync(0xffffffffu, ok) | 1u);
        const uint32_t nlo = lo + m * stride;
        hi = min(hi, nlo + stride);
        lo = nlo;
    }
    return lo;
}

__global__ void k_buf_init(medusa_buf_report* rep) {
    pdl_wait();  // the previous user of the report may still read it
    pdl_trigger();
    rep->n_bad = 0;
    rep->first_bad = ~0ull;
}

// One warp per 2 KB task of the blob (lane l owns the 16-byte units l, l+32,
// l+64, l+96 of the task).  The warp keeps a window of 32 consecutive segment
// descriptors {start, end, target address, valid} in shared memory, starting
// at the segment that holds the task's first byte; units inside the window are
// resolved by a 5-step search in shared memory, tasks that span more than 32
// segments slide the window.  A unit inside one segment whose target address
// is 16-byte aligned moves as one 16-byte load + store (all four loads of a
// lane are issued before its stores); anything else goes byte by byte.
template <bool kToBlob>
__global__ void __launch_bounds__(kCopyThreads, 4)
k_buf_copy(uint8_t* blob_w, const uint8_t* __restrict__ blob_r, const uint32_t* __restrict__ perm,
           const uint64_t* __restrict__ off, uint32_t n_perm, const uint64_t* __restrict__ base,
           const uint64_t* __restrict__ size, uint32_t n_alloc, medusa_buf_report* rep) {
    constexpr int kUnits = kTaskBytes / 16 / 32;  // units per lane per task (4)
    __shared__ uint64_t s_s[kCopyThreads], s_e[kCopyThreads], s_a[kCopyThreads];
    __shared__ uint32_t s_ok[kCopyThreads / 32];
    const uint32_t lane = threadIdx.x & 31, wslot = threadIdx.x & ~31u;
    const uint64_t gtid = (uint64_t)blockIdx.x * kCopyThreads + threadIdx.x;
    const uint64_t nthreads = (uint64_t)gridDim.x * kCopyThreads;
    uint64_t* ws = s_s + wslot;
    uint64_t* we = s_e + wslot;
    uint64_t* wa = s_a + wslot;
    if (n_perm > 0) {
        // 1. the copy: warp w moves the contiguous blob range [w*per, (w+1)*per)
        //    in batches of 2 KB; its descriptor window slides along the range
        const uint64_t total = __ldg(off + n_perm);
        const uint64_t nwarps = nthreads >> 5;
        const uint64_t per = ((total + nwarps - 1) / nwarps + kTaskBytes - 1) / kTaskBytes * kTaskBytes;
        const uint64_t r0 = (gtid >> 5) * per, r1 = min(r0 + per, total);
        // window of descriptors k .. k+31 (one per lane) into this warp's shared slice
        auto load_window = [&](uint32_t k) {
            const uint64_t kk = (uint64_t)k + lane;
            uint64_t ss = total, ee = total, aa = 0;
            bool ok = false;
            if (kk < n_perm) {
                ss = __ldg(off + kk);
                ee = __ldg(off + kk + 1);
                const uint32_t id = __ldg(perm + kk);
                if (id < n_alloc) {
                    aa = __ldg(base + id);
                    ok = !size || ee - ss <= __ldg(size + id);
                }
            }
            __syncwarp();
            ws[lane] = ss;
            we[lane] = ee;
            wa[lane] = aa;
            const uint32_t okm = __ballot_sync(0xffffffffu, ok);
            if (lane == 0) s_ok[threadIdx.x >> 5] = okm;
            __syncwarp();
        };
        if (r0 < r1) {
            // the segment holding r0: one probe of 32 offsets around the index a
            // uniform segment size predicts (one round when the guess is close, as
            // for equally sized buffers); else the 32-ary search
            uint32_t k;
            {
                const uint64_t guess = (uint64_t)((double)r0 / (double)total * (double)n_perm);
                const uint32_t g0 = (uint32_t)min(guess > 8 ? guess - 8 : (uint64_t)0, (uint64_t)(n_perm > 32 ? n_perm - 32 : 0));
                const uint32_t kk = g0 + lane;
                const bool le = kk < n_perm && __ldg(off + kk) <= r0;
                const uint32_t b = __ballot_sync(0xffffffffu, le);
                // bracketed: off[g0] <= r0 and (the probe ends past r0, or it reaches n_perm)
                const bool hit_lo = b & 1u;
                const bool hit_hi = (b != 0xffffffffu) || g0 + 32 >= n_perm;
                k = (hit_lo && hit_hi) ? g0 + 31 - __clz(b) : warp_last_le(off, 0, n_perm, r0);
            }
            load_window(k);
            for (uint64_t t0 = r0; t0 < r1; t0 += kTaskBytes) {
                const uint64_t t1 = min(t0 + kTaskBytes, r1);
                uint64_t q_next[kUnits];  // next byte of each unit still to move (>= unit end: done)
#pragma unroll
                for (int r = 0; r < kUnits; ++r) q_next[r] = t0 + 16ull * (lane + 32 * r);
                while (true) {
                    const uint64_t w_end = we[31];  // bytes below w_end are covered by the window
                    const uint32_t okm = s_ok[threadIdx.x >> 5];
                    auto find = [&](uint64_t q) {  // last j with start <= q (q inside the window)
                        uint32_t j = 0;
#pragma unroll
                        for (int b = 16; b >= 1; b >>= 1)
                            if (ws[j + b] <= q) j += b;  // j + b <= 31
                        return j;
                    };
                    // fast path: whole unit inside one valid segment, aligned target.
                    // The four units' segment searches run interleaved (independent
                    // shared-memory chains), then all loads are issued, then the stores.
                    uint4 v[kUnits];
                    uint64_t dst_a[kUnits];
                    bool fast[kUnits];
                    uint32_t jr[kUnits];
#pragma unroll
                    for (int r = 0; r < kUnits; ++r) jr[r] = 0;
#pragma unroll
                    for (int b = 16; b >= 1; b >>= 1) {
#pragma unroll
                        for (int r = 0; r < kUnits; ++r) {
                            const uint64_t p = t0 + 16ull * (lane + 32 * r);
                            if (ws[jr[r] + b] <= p) jr[r] += b;  // jr + b <= 31
                        }
                    }
#pragma unroll
                    for (int r = 0; r < kUnits; ++r) {
                        const uint64_t p = t0 + 16ull * (lane + 32 * r);
                        fast[r] = false;
                        if (q_next[r] != p || p >= t1 || p >= w_end) continue;
                        const uint32_t j = jr[r];
                        if (p + 16 > we[j]) continue;
                        const uint64_t a = wa[j] + (p - ws[j]);
                        if ((a & 15) != 0) continue;
                        if (!((okm >> j) & 1)) {  // invalid segment: nothing to move
                            q_next[r] = ~0ull;
                            continue;
                        }
                        fast[r] = true;
                        if (kToBlob) {
                            v[r] = __ldg(reinterpret_cast<const uint4*>(a));
                            dst_a[r] = reinterpret_cast<uint64_t>(blob_w + p);
                        } else {
                            v[r] = __ldg(reinterpret_cast<const uint4*>(blob_r + p));
                            dst_a[r] = a;
                        }
                    }
#pragma unroll
                    for (int r = 0; r < kUnits; ++r) {
                        if (!fast[r]) continue;
                        *reinterpret_cast<uint4*>(dst_a[r]) = v[r];
                        q_next[r] = ~0ull;
                    }
                    // byte path for the rest, inside this window
                    bool more = false;
#pragma unroll
                    for (int r = 0; r < kUnits; ++r) {
                        const uint64_t p = t0 + 16ull * (lane + 32 * r);
                        const uint64_t u_end = min(p + 16, t1);
                        uint64_t q = q_next[r];
                        for (; q < u_end && q < w_end; ++q) {
                            const uint32_t j = find(q);
                            if (q >= we[j] || !((okm >> j) & 1)) continue;  // empty tail / invalid segment
                            const uint64_t a = wa[j] + (q - ws[j]);
                            if (kToBlob) blob_w[q] = *reinterpret_cast<const uint8_t*>(a);
                            else *reinterpret_cast<uint8_t*>(a) = blob_r[q];
                        }
                        q_next[r] = q;
                        more |= q < u_end;
                    }
                    if (!__any_sync(0xffffffffu, more)) break;
                    k += 32;  // every byte below w_end is done: the next 32 segments
                    load_window(k);
                }
            }
        }
    }
    // 2. validation (R-B4), counted once per segment: a segment whose allocation
    //    the replay did not make, or that is longer than the replayed allocation,
    //    was not copied.  (After the copy: its loads overlap the stores draining.)
    uint32_t n_bad = 0;
    uint64_t first = ~0ull;
    for (uint64_t k = gtid; k < n_perm; k += nthreads) {
        const uint32_t id = perm[k];
        if (id >= n_alloc || (size && off[k + 1] - off[k] > size[id])) {
            ++n_bad;
            first = min(first, k);
        }
    }
    pdl_wait();  // k_buf_init has initialised the report
    pdl_trigger();
    if (n_bad) {
        atomicAdd(reinterpret_cast<unsigned long long*>(&rep->n_bad), (unsigned long long)n_bad);
        atomicMin(reinterpret_cast<unsigned long long*>(&rep->first_bad), (unsigned long long)first);
    }
}

}  // namespace

medusa_status run_buffers_plan(const medusa_alloc* alloc, uint32_t n_alloc, const uint32_t* cap, uint32_t n_cap,
                               const uint64_t* slot, uint64_t n_slots, uint8_t* cls, uint32_t* perm,
                               uint64_t* perm_off, uint32_t capacity, uint32_t* h_n_perm, uint64_t* h_bytes,
                               cudaStream_t stream, cudaError_t* err) {
    const uint32_t n_tiles = (n_alloc + kTile - 1) / kTile;
    void* scratch = nullptr;
    const size_t sbytes = sizeof(PlanResult) + (size_t)std::max(n_tiles, 1u) * (sizeof(uint32_t) + sizeof(uint64_t));
    cudaError_t e = cudaMallocAsync(&scratch, sbytes, stream);
    if (e != cudaSuccess) { *err = e; return MEDUSA_ERR_CUDA; }
    PlanResult* res = static_cast<PlanResult*>(scratch);
    uint64_t* tile_bytes = reinterpret_cast<uint64_t*>(res + 1);
    uint32_t* tile_cnt = reinterpret_cast<uint32_t*>(tile_bytes + std::max(n_tiles, 1u));
    PlanResult h{};
    do {
        if ((e = cudaMemsetAsync(res, 0, sizeof(PlanResult), stream)) != cudaSuccess) break;
        if (n_alloc > 0) {
            if ((e = cudaMemsetAsync(cls, 0, n_alloc, stream)) != cudaSuccess) break;
            if (n_slots > 0) {
                TimedLaunch tl("buf_mark", stream);
                const uint64_t want = (n_slots + kPlanThreads - 1) / kPlanThreads;
                const unsigned grid = (unsigned)std::min<uint64_t>(want, 148ull * 8);
                k_buf_mark<<<grid, kPlanThreads, 0, stream>>>(slot, n_slots, n_alloc, cls);
                if ((e = cudaGetLastError()) != cudaSuccess) break;
            }
            {
                TimedLaunch tl("buf_class", stream);
                k_buf_class<<<n_tiles, kPlanThreads, 0, stream>>>(alloc, n_alloc, cap, n_cap, cls, tile_cnt,
                                                                  tile_bytes, res);
                if ((e = cudaGetLastError()) != cudaSuccess) break;
            }
            {
                TimedLaunch tl("buf_scatter", stream);
                k_buf_scatter<<<n_tiles, kPlanThreads, 0, stream>>>(alloc, n_alloc, cls, tile_cnt, tile_bytes,
                                                                    n_tiles, perm, perm_off, capacity, res);
                if ((e = cudaGetLastError()) != cudaSuccess) break;
            }
        } else {
            // no allocation: still check the capture intervals, offsets = {0}
            k_buf_class<<<1, kPlanThreads, 0, stream>>>(alloc, 0, cap, n_cap, cls, tile_cnt, tile_bytes, res);
            if ((e = cudaGetLastError()) != cudaSuccess) break;
            if (perm_off && (e = cudaMemsetAsync(perm_off, 0, 8, stream)) != cudaSuccess) break;
        }
        if ((e = cudaMemcpyAsync(&h, res, sizeof(h), cudaMemcpyDeviceToHost, stream)) != cudaSuccess) break;
        e = cudaFreeAsync(scratch, stream);
        scratch = nullptr;
        if (e != cudaSuccess) break;
        e = cudaStreamSynchronize(stream);
    } while (0);
    if (scratch) cudaFreeAsync(scratch, stream);
    if (e != cudaSuccess) { *err = e; return MEDUSA_ERR_CUDA; }
    if (h.bad_capture) return MEDUSA_ERR_INVALID_ARG;
    *h_n_perm = (uint32_t)h.n_perm;
    *h_bytes = h.bytes;
    return h.n_perm > capacity ? MEDUSA_ERR_CAPACITY : MEDUSA_OK;
}

cudaError_t launch_buffers_copy(bool to_blob, uint8_t* blob_w, const uint8_t* blob_r, const uint32_t* perm,
                                const uint64_t* perm_off, uint32_t n_perm, const uint64_t* base, const uint64_t* size,
                                uint32_t n_alloc, medusa_buf_report* rep, cudaStream_t stream) {
    int dev = 0, n_sm = 148, per_sm = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n_sm, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, to_blob ? k_buf_copy<true> : k_buf_copy<false>,
                                                  kCopyThreads, 0);
    const unsigned grid = (unsigned)n_sm * (unsigned)std::max(per_sm, 1);  // persistent: one wave
    cudaError_t e;
    {
        TimedLaunch tl("buf_report_init", stream);
        if ((e = launch_pdl(k_buf_init, 1, 1, 0, stream, rep)) != cudaSuccess) return e;
    }
    if (to_blob) {
        TimedLaunch tl("buf_save", stream);
        e = launch_pdl(k_buf_copy<true>, grid, kCopyThreads, 0, stream, blob_w, (const uint8_t*)nullptr, perm,
                       perm_off, n_perm, base, (const uint64_t*)nullptr, n_alloc, rep);
    } else {
        TimedLaunch tl("buf_restore", stream);
        e = launch_pdl(k_buf_copy<false>, grid, kCopyThreads, 0, stream, (uint8_t*)nullptr, blob_r, perm,
                       perm_off, n_perm, base, size, n_alloc, rep);
    }
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace medusa
