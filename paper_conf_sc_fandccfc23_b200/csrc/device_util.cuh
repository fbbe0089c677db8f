// device_util.cuh — small device helpers shared by the sweep kernels (no method arithmetic).
#pragma once
#include <cuda_runtime.h>
#include <math_constants.h>
#include <climits>
#include <cstdint>

#include "internal.h"

namespace syn {

// 32-bit shared-memory addressing (keeps the hot loops free of generic-address conversions)
__device__ __forceinline__ unsigned su32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ float lds_f(unsigned a) {
    float v;
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ unsigned lds_u(unsigned a) {
    unsigned v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_f(unsigned a, float v) { asm volatile("st.shared.f32 [%0], %1;" :: "r"(a), "f"(v)); }
__device__ __forceinline__ void sts_u(unsigned a, unsigned v) { asm volatile("st.shared.u32 [%0], %1;" :: "r"(a), "r"(v)); }

// Whole 32-byte 2-level block in one 256-bit load (sm_100: LDG.E.ENL2.256), one L1 request per
// block; blocks are 32-byte aligned and immutable for the kernel's lifetime (read-only path).
__device__ __forceinline__ void ldg_blk256(const uint4* p, uint4& A, uint4& B) {
    asm volatile("ld.global.nc.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=r"(A.x), "=r"(A.y), "=r"(A.z), "=r"(A.w), "=r"(B.x), "=r"(B.y), "=r"(B.z), "=r"(B.w)
                 : "l"(p));
}

__device__ __forceinline__ uint2 ldg_node(const uint2* p) {
    uint2 r;
    asm volatile("ld.global.nc.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
    return r;
}

// Model m of a call: 0 speedup, 1 energy, 2 direct EDP, 3 direct ED2P (four-model variant).
__device__ __forceinline__ const DevModel& model_of(const SweepArgs& a, int m) {
    return m == 0 ? a.ms : m == 1 ? a.me : a.mx[m - 2];
}

__device__ __forceinline__ bool model_present(const SweepArgs& a, int m) { return m < 2 || a.has_x[m - 2]; }

// Trees of model m's forest member (0 without one).
__device__ __forceinline__ int trees_of(const SweepArgs& a, int m) {
    if (!model_present(a, m)) return 0;
    const DevModel& d = model_of(a, m);
    return d.forest_weight != 0.0 ? d.n_trees : 0;
}

}  // namespace syn
