// peaks.cu — measurement tool: on-chip throughput ceilings for the k_tm_walk roofline.
//
// NOT part of the product library.  bench.py calls peaks_measure() once per run, on the GPU it
// benchmarks, to get measured denominators for the on-chip roofline (MEASURED_PEAKS.json holds
// only HBM and tensor-core figures):
//   l1_scatter32  scattered, independent 32-byte loads (one 256-bit LDG.E.ENL2.256 each, the
//                 k_tm_walk block fetch) from a per-SM window that stays resident in L1: bytes/s,
//                 requests/s and requests per clock per SM
//   l2_scatter32  the same loads over a 16 MB window (L1 misses, L2 hits)
//   smem_read     conflict-free 128-bit shared-memory loads: bytes/s and bytes per clock per SM
// Each kernel runs on every SM with 2 CTAs x 512 threads (k_tm_walk's shape), many loads in
// flight per thread, timed with CUDA events (best of 5); clock64() spans give the per-clock view.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

namespace {

__device__ __forceinline__ void ldg256(const uint4* p, uint4& A, uint4& B) {
    asm volatile("ld.global.nc.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=r"(A.x), "=r"(A.y), "=r"(A.z), "=r"(A.w), "=r"(B.x), "=r"(B.y), "=r"(B.z), "=r"(B.w)
                 : "l"(p));
}

// window_blocks: power of two, number of 32-B blocks each CTA draws from (offset per SM pair)
__global__ void __launch_bounds__(512, 2) k_scatter32(const uint4* __restrict__ buf, unsigned window_blocks,
                                                      unsigned long long stride_blocks, int iters,
                                                      unsigned* sink, long long* cycles) {
    const uint4* base = buf + 2ull * (unsigned long long)(blockIdx.x >> 1) * stride_blocks;
    unsigned x = (threadIdx.x + 1u) * 2654435761u ^ (blockIdx.x * 40503u);
    unsigned acc = 0;
    __syncthreads();
    const long long t0 = clock64();
#pragma unroll 8
    for (int i = 0; i < iters; ++i) {
        x = x * 1664525u + 1013904223u;
        const unsigned b = (x >> 7) & (window_blocks - 1u);
        uint4 A, B;
        ldg256(base + 2ull * b, A, B);
        acc ^= A.x ^ B.w;
    }
    __syncthreads();
    const long long t1 = clock64();
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

// W consecutive 32-byte pieces per load (W = 1, 2, 4: 32 / 64 / 128 bytes, one 128-byte line at
// most) from random W-aligned positions of the window: is a wider block cheaper per byte?
template <int W>
__global__ void __launch_bounds__(512, 2) k_scatter_w(const uint4* __restrict__ buf, unsigned window_blocks,
                                                      unsigned long long stride_blocks, int iters,
                                                      unsigned* sink, long long* cycles) {
    const uint4* base = buf + 2ull * (unsigned long long)(blockIdx.x >> 1) * stride_blocks;
    unsigned x = (threadIdx.x + 1u) * 2654435761u ^ (blockIdx.x * 40503u);
    unsigned acc = 0;
    __syncthreads();
    const long long t0 = clock64();
#pragma unroll 4
    for (int i = 0; i < iters; ++i) {
        x = x * 1664525u + 1013904223u;
        const unsigned b = ((x >> 7) & (window_blocks - 1u)) & ~(unsigned)(W - 1);
#pragma unroll
        for (int w = 0; w < W; ++w) {
            uint4 A, B;
            ldg256(base + 2ull * (b + w), A, B);
            acc ^= A.x ^ B.w;
        }
    }
    __syncthreads();
    const long long t1 = clock64();
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

// Lane pairs: lanes 2i and 2i+1 load the two 32-byte halves of one 64-byte aligned region in the
// same instruction (one line per pair), as two lanes sharing 64-byte blocks would.
__global__ void __launch_bounds__(512, 2) k_scatter_pair(const uint4* __restrict__ buf, unsigned window_blocks,
                                                         unsigned long long stride_blocks, int iters,
                                                         unsigned* sink, long long* cycles) {
    const uint4* base = buf + 2ull * (unsigned long long)(blockIdx.x >> 1) * stride_blocks;
    unsigned x = ((threadIdx.x >> 1) + 1u) * 2654435761u ^ (blockIdx.x * 40503u);
    unsigned acc = 0;
    __syncthreads();
    const long long t0 = clock64();
#pragma unroll 8
    for (int i = 0; i < iters; ++i) {
        x = x * 1664525u + 1013904223u;
        const unsigned b = (((x >> 7) & (window_blocks - 1u)) & ~1u) + (threadIdx.x & 1u);
        uint4 A, B;
        ldg256(base + 2ull * b, A, B);
        acc ^= A.x ^ B.w;
    }
    __syncthreads();
    const long long t1 = clock64();
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

__global__ void __launch_bounds__(512, 2) k_smem_read(int iters, unsigned* sink, long long* cycles) {
    extern __shared__ uint4 sm[];                       // 512 x 16 B per CTA (8 KB)
    sm[threadIdx.x] = make_uint4(threadIdx.x, threadIdx.x * 3u, threadIdx.x * 5u, threadIdx.x * 7u);
    __syncthreads();
    const unsigned a = (unsigned)__cvta_generic_to_shared(sm);
    unsigned acc = 0;
    unsigned idx = threadIdx.x;
    const long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < iters; ++i) {
        uint4 v;
        asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                     : "r"(a + 16u * idx));
        acc ^= v.x ^ v.w;
        idx = (idx + 32u) & 511u;                       // each warp reads 32 consecutive 16-B words
    }
    __syncthreads();
    const long long t1 = clock64();
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

template <typename L>
float best_ms(L launch, int reps) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    launch();                                           // warm-up (fills L1 / L2)
    float best = 1e30f;
    for (int r = 0; r < reps; ++r) {
        cudaEventRecord(a);
        launch();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = 0.0f;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    return best;
}

double mean_cycles(const long long* d, int n) {
    long long h[4096];
    cudaMemcpy(h, d, sizeof(long long) * n, cudaMemcpyDeviceToHost);
    double s = 0.0;
    for (int i = 0; i < n; ++i) s += (double)h[i];
    return s / n;
}

}  // namespace

extern "C" {

// out[0..8]: l1 bytes/s, l1 requests/s, l1 requests per clk per SM, l2 bytes/s, l2 requests/s,
// smem bytes/s, smem bytes per clk per SM, SMs, kernel clock (MHz, from clock64 / event time).
// Returns 0, or a CUDA error code.
int peaks_measure(int device, double* out) {
    if (cudaSetDevice(device) != cudaSuccess) return 1;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    const int ctas = 2 * sms, nt = 512;
    const unsigned l1_window = 2048;                     // 64 KB per SM: L1-resident
    const unsigned l2_window = 1u << 19;                 // 16 MB shared by all SMs: L2-resident
    uint4* buf = nullptr;
    unsigned* sink = nullptr;
    long long* cyc = nullptr;
    const size_t bytes = std::max<size_t>((size_t)(ctas / 2) * l1_window * 32, (size_t)l2_window * 32);
    if (cudaMalloc(&buf, bytes) != cudaSuccess || cudaMalloc(&sink, 4) != cudaSuccess ||
        cudaMalloc(&cyc, sizeof(long long) * ctas) != cudaSuccess)
        return 2;
    cudaMemset(buf, 1, bytes);
    const int iters = 4096;
    const double loads = (double)ctas * nt * iters;
    float ms = best_ms([&] { k_scatter32<<<ctas, nt>>>(buf, l1_window, l1_window, iters, sink, cyc); }, 5);
    const double c1 = mean_cycles(cyc, ctas);
    out[0] = loads * 32.0 / (ms * 1e-3);
    out[1] = loads / (ms * 1e-3);
    out[2] = loads / sms / c1;                           // requests per clock per SM (CTA-span clocks)
    out[8] = c1 / (ms * 1e-3) / 1e6;
    ms = best_ms([&] { k_scatter32<<<ctas, nt>>>(buf, l2_window, 0, iters / 4, sink, cyc); }, 5);
    out[3] = loads / 4 * 32.0 / (ms * 1e-3);
    out[4] = loads / 4 / (ms * 1e-3);
    const int siters = 16384;
    ms = best_ms([&] { k_smem_read<<<ctas, nt, nt * 16>>>(siters, sink, cyc); }, 5);
    const double c3 = mean_cycles(cyc, ctas);
    out[5] = (double)ctas * nt * siters * 16.0 / (ms * 1e-3);
    out[6] = (double)ctas * nt * siters * 16.0 / sms / c3;
    out[7] = sms;
    cudaError_t e = cudaGetLastError();
    cudaFree(buf);
    cudaFree(sink);
    cudaFree(cyc);
    return e == cudaSuccess ? 0 : (int)e;
}

// Scattered loads of `width` bytes (32, 64, 128; 1 = 32-byte halves of 64-byte regions by lane pairs) over a window of `window_blocks` 32-byte blocks
// per SM (L1-resident when small): out[0] = bytes/s, out[1] = loads/s (one load = width bytes).
int peaks_scatter(int device, int width, unsigned window_blocks, int iters, double* out) {
    if (cudaSetDevice(device) != cudaSuccess) return 1;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    const int ctas = 2 * sms, nt = 512;
    uint4* buf = nullptr;
    unsigned* sink = nullptr;
    long long* cyc = nullptr;
    const size_t bytes = (size_t)(ctas / 2 + 1) * window_blocks * 32;
    if (cudaMalloc(&buf, bytes) != cudaSuccess || cudaMalloc(&sink, 4) != cudaSuccess ||
        cudaMalloc(&cyc, sizeof(long long) * ctas) != cudaSuccess)
        return 2;
    cudaMemset(buf, 1, bytes);
    float ms = 0.0f;
    if (width == 32) ms = best_ms([&] { k_scatter_w<1><<<ctas, nt>>>(buf, window_blocks, window_blocks, iters, sink, cyc); }, 5);
    else if (width == 64) ms = best_ms([&] { k_scatter_w<2><<<ctas, nt>>>(buf, window_blocks, window_blocks, iters, sink, cyc); }, 5);
    else if (width == 128) ms = best_ms([&] { k_scatter_w<4><<<ctas, nt>>>(buf, window_blocks, window_blocks, iters, sink, cyc); }, 5);
    else ms = best_ms([&] { k_scatter_pair<<<ctas, nt>>>(buf, window_blocks, window_blocks, iters, sink, cyc); }, 5);   // 2 lanes / 64 B
    if (width == 1) width = 32;
    const double loads = (double)ctas * nt * iters;
    out[0] = loads * width / (ms * 1e-3);
    out[1] = loads / (ms * 1e-3);
    cudaError_t e = cudaGetLastError();
    cudaFree(buf);
    cudaFree(sink);
    cudaFree(cyc);
    return e == cudaSuccess ? 0 : (int)e;
}

}  // extern "C"
