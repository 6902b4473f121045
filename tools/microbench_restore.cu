// Micro-benchmark (not part of the library): what does each ingredient of the
// restore pass cost on B200?  25 MB image, 2048-word chunks, ~18% slots.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb tools/microbench_restore.cu && ./mb
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

constexpr int CW = 2048;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k_copy(const uint4* __restrict__ s, uint4* __restrict__ d, size_t n16) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) d[i] = s[i];
}

template <int MODE>  // 0: TMA in/out, 1: + records, 2: + records + gathers, 3: + apply (full)
__global__ void __launch_bounds__(128) k_tma(const uint64_t* src, uint64_t* dst, size_t n_words, const uint32_t* cb,
                                             const uint64_t* rec, const uint64_t* b0, const uint64_t* b1, const uint64_t* b2,
                                             unsigned long long* sink) {
    __shared__ __align__(128) uint64_t w[CW];
    __shared__ __align__(8) unsigned long long mbar;
    const uint32_t c = blockIdx.x, tid = threadIdx.x;
    const uint32_t mb = su32(&mbar);
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(CW * 8) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(su32(w)), "l"(src + (size_t)c * CW), "r"(CW * 8), "r"(mb) : "memory");
    }
    uint64_t acc = 0;
    if (MODE >= 1) {
        const uint32_t r0 = cb[c], r1 = cb[c + 1];
        for (uint32_t r = r0 + tid; r < r1; r += 128) {
            const uint64_t x = rec[r];
            if (MODE >= 2) {
                const uint64_t id = x >> 40;
                acc += b0[id] + b1[id] + b2[id];
            } else {
                acc += x;
            }
        }
    }
    __syncthreads();
    uint32_t ready = 0;
    while (!ready)
        asm volatile("{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], 0; selp.u32 %0, 1, 0, P; }"
                     : "=r"(ready) : "r"(mb) : "memory");
    if (MODE >= 3 && acc) w[tid] += acc & 1;  // touch shared words (data dependent)
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (tid == 0) {
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + (size_t)c * CW), "r"(su32(w)),
                     "r"(CW * 8) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    }
    if (acc == 0x123456789ull) *sink = acc;
}

int main() {
    const size_t n_words = 3096576;  // 1512 chunks
    const uint32_t C = n_words / CW;
    const size_t n_alloc = 199146;
    uint64_t *src, *dst, *rec, *b0, *b1, *b2;
    uint32_t* cb;
    unsigned long long* sink;
    char* scrub;
    CK(cudaMalloc(&src, n_words * 8)); CK(cudaMalloc(&dst, n_words * 8));
    CK(cudaMalloc(&rec, n_words * 8)); CK(cudaMalloc(&cb, (C + 1) * 4));
    CK(cudaMalloc(&b0, n_alloc * 8)); CK(cudaMalloc(&b1, n_alloc * 8)); CK(cudaMalloc(&b2, n_alloc * 8));
    CK(cudaMalloc(&sink, 8)); CK(cudaMalloc(&scrub, 512 << 20));
    std::vector<uint32_t> hcb(C + 1);
    for (uint32_t c = 0; c <= C; ++c) hcb[c] = c * 383;
    std::vector<uint64_t> hrec(C * 383 + 1);
    uint64_t st = 88172645463325252ull;
    for (auto& r : hrec) { st ^= st << 13; st ^= st >> 7; st ^= st << 17; r = ((st % n_alloc) << 40) | (st & 0xFFFF); }
    CK(cudaMemcpy(cb, hcb.data(), (C + 1) * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(rec, hrec.data(), hrec.size() * 8, cudaMemcpyHostToDevice));
    CK(cudaMemset(src, 1, n_words * 8));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    const double bytes = 2.0 * n_words * 8;
    auto run = [&](const char* name, auto launch, bool flush) {
        for (int i = 0; i < 3; ++i) launch();
        float tot = 0;
        const int reps = 20;
        for (int i = 0; i < reps; ++i) {
            if (flush) CK(cudaMemsetAsync(scrub, i, 512 << 20));
            cudaEventRecord(e0);
            launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1); tot += ms;
        }
        CK(cudaGetLastError());
        const double us = tot / reps * 1e3;
        printf("%-34s %s %8.2f us  %7.0f GB/s (copy bytes)\n", name, flush ? "cold" : "warm", us, bytes / us / 1e3);
    };
    for (int flush = 1; flush >= 0; --flush) {
        for (int g : {148 * 4, 148 * 8, 148 * 16})
            run(g == 592 ? "plain copy 16B grid=592" : (g == 1184 ? "plain copy 16B grid=1184" : "plain copy 16B grid=2368"),
                [&] { k_copy<<<g, 256>>>((const uint4*)src, (uint4*)dst, n_words / 2); }, flush);
        run("cudaMemcpyAsync D2D", [&] { cudaMemcpyAsync(dst, src, n_words * 8, cudaMemcpyDeviceToDevice); }, flush);
        run("TMA in/out per chunk", [&] { k_tma<0><<<C, 128>>>(src, dst, n_words, cb, rec, b0, b1, b2, sink); }, flush);
        run("TMA + records", [&] { k_tma<1><<<C, 128>>>(src, dst, n_words, cb, rec, b0, b1, b2, sink); }, flush);
        run("TMA + records + gathers", [&] { k_tma<2><<<C, 128>>>(src, dst, n_words, cb, rec, b0, b1, b2, sink); }, flush);
        run("TMA + records + gathers + apply", [&] { k_tma<3><<<C, 128>>>(src, dst, n_words, cb, rec, b0, b1, b2, sink); }, flush);
    }
    return 0;
}
