// kernels_svr.cuh — SVR_RBF member over a clock sweep (Table 2; Q24).
//
// With z = (x - mean) / scale the squared distance of (kernel k, clock f_i) to support vector j
// splits into a static-feature part and a clock part,
//   ||z(k, f_i) - sv_j||^2 = A_kj + B_ji,  A_kj = sum_{d<F} (z_kd - sv_jd)^2,  B_ji = (z(f_i) - sv_jF)^2,
// so svr(k, f_i) = b + sum_j U_kj V_ji with U_kj = dual_j e^{-gamma A_kj}, V_ji = e^{-gamma B_ji}:
// an fp64 [n_k x n_sv] x [n_sv x n_f] contraction.  tcgen05 has no fp64 kind, so the contraction
// runs on the fp64 FMA pipe:
//   k_svr_v  V once per call, tiled [clock tile][SV][tn] so a k_svr chunk is one contiguous block
//   k_svr_u  U per kernel slab, tiled [kernel tile][SV][64] (one exp per (k, j))
//   k_svr    each thread an 8-kernel x CPT-clock register tile; U/V chunks of 16 SVs arrive by
//            1-D bulk copies (cp.async.bulk + mbarrier, 3-stage ring); SV ranges split across
//            CTAs (blockIdx.z) when the batch is too small to fill the GPU
// finish_tile sums the split partials in split order, adds the intercept and the member
// (add_svr_unit).
#pragma once
#include "internal.h"

namespace syn {

__device__ __forceinline__ unsigned svr_su32(const void* p) {
    return (unsigned)__cvta_generic_to_shared(p);
}

// V tiles: Vt[it][j][c] = exp(-gamma * (z(f_i) - sv[j][F])^2), i = it * tn + c; zero padding
__global__ void __launch_bounds__(256) k_svr_v(const __grid_constant__ SvrArgs a) {
    const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long per_tile = (long long)a.n_svp * a.tn;
    const int tiles_n = (a.n_f + a.tn - 1) / a.tn;
    if (t >= per_tile * tiles_n) return;
    const int it = (int)(t / per_tile);
    const long long r = t - it * per_tile;
    const int j = (int)(r / a.tn), c = (int)(r - (long long)j * a.tn);
    const int i = it * a.tn + c;
    const int F = a.F;
    double v = 0.0;
    if (j < a.n_sv && i < a.n_f) {
        const double zc = __ddiv_rn(__dsub_rn((double)__ldg(a.freqs + i), __ldg(a.in_mean + F)), __ldg(a.in_scale + F));
        const double b = __dsub_rn(zc, (double)__ldg(a.sv + (size_t)j * (F + 1) + F));
        v = exp(-__dmul_rn(a.gamma, __dmul_rn(b, b)));
    }
    a.Vt[t] = v;
}

// U tiles for kernel tile blockIdx.x of the slab and SVs [kSvrJC * blockIdx.y, +kSvrJC):
//   Ut[kt][j][kk] = dual_j * exp(-gamma * sum_{d<F} (z_kd - sv_jd)^2); zero padding.
// 256 threads = 64 kernels x 4 SV lanes, 4 independent SVs per thread (ILP across the exps).
__global__ void __launch_bounds__(256) k_svr_u(const __grid_constant__ SvrArgs a) {
    extern __shared__ __align__(16) double svu[];
    const int F = a.F;
    double* z = svu;                                        // [F][64]
    float* s = reinterpret_cast<float*>(z + (size_t)F * 64); // [F][kSvrJC]
    const int kt = blockIdx.x, j0 = blockIdx.y * kSvrJC;
    const long long kb = a.slab0 + (long long)kt * kSvrTK;
    const int nk = (int)min((long long)kSvrTK, a.slab0 + a.nks - kb);
    const int nj = min(kSvrJC, a.n_sv - j0);
    for (int e = threadIdx.x; e < kSvrTK * F; e += 256) {
        const int kk = e / F, d = e - kk * F;
        double v = 0.0;
        if (kk < nk)
            v = __ddiv_rn(__dsub_rn((double)__ldg(a.features + kb * F + e), __ldg(a.in_mean + d)), __ldg(a.in_scale + d));
        z[d * 64 + kk] = v;
    }
    for (int e = threadIdx.x; e < kSvrJC * F; e += 256) {
        const int q = e / F, d = e - q * F;
        s[d * kSvrJC + q] = q < nj ? __ldg(a.sv + (size_t)(j0 + q) * (F + 1) + d) : 0.0f;
    }
    __syncthreads();
    const int kk = threadIdx.x & 63, q0 = threadIdx.x >> 6;
    constexpr int R = kSvrJC / 4;
    double A[R];
#pragma unroll
    for (int r = 0; r < R; ++r) A[r] = 0.0;
    for (int d = 0; d < F; ++d) {
        const double zk = z[d * 64 + kk];
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const double t = __dsub_rn(zk, (double)s[d * kSvrJC + q0 + 4 * r]);
            A[r] = __dadd_rn(A[r], __dmul_rn(t, t));
        }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int q = q0 + 4 * r;
        const double val = (kk < nk && q < nj) ? __dmul_rn(__ldg(a.dual + j0 + q), exp(-__dmul_rn(a.gamma, A[r]))) : 0.0;
        a.Ut[((size_t)kt * a.n_svp + j0 + q) * kSvrTK + kk] = val;
    }
}

__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(svr_su32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(svr_su32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned phase) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "SVR_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra SVR_WAIT_%=;\n}" ::"r"(svr_su32(bar)), "r"(phase) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, unsigned long long* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(svr_su32(dst)), "l"(src), "r"(bytes), "r"(svr_su32(bar)) : "memory");
}

template <int CPT>
__global__ void __launch_bounds__(256, 1) k_svr(const __grid_constant__ SvrArgs a) {
    extern __shared__ __align__(128) double svm[];
    constexpr int TN = 32 * CPT;
    constexpr unsigned UB = kSvrJC * kSvrTK * 8, VB = kSvrJC * TN * 8;
    double* Ub = svm;                                       // [stages][JC][TK]
    double* Vb = Ub + kSvrStages * kSvrJC * kSvrTK;         // [stages][JC][TN]
    unsigned long long* bar = reinterpret_cast<unsigned long long*>(Vb + kSvrStages * kSvrJC * TN);
    const int kt = blockIdx.x, it = blockIdx.y;
    const int c_beg = blockIdx.z * a.chunks_per_split;
    const int nch = min(a.chunks_per_split, a.n_svp / kSvrJC - c_beg);
    const double* ug = a.Ut + ((size_t)kt * a.n_svp + (size_t)c_beg * kSvrJC) * kSvrTK;
    const double* vg = a.Vt + ((size_t)it * a.n_svp + (size_t)c_beg * kSvrJC) * TN;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int q = 0; q < kSvrStages; ++q) mbar_init(bar + q, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int c = 0; c < min(kSvrStages - 1, nch); ++c) {
            mbar_expect_tx(bar + c, UB + VB);
            bulk_g2s(Ub + (size_t)c * kSvrJC * kSvrTK, ug + (size_t)c * kSvrJC * kSvrTK, UB, bar + c);
            bulk_g2s(Vb + (size_t)c * kSvrJC * TN, vg + (size_t)c * kSvrJC * TN, VB, bar + c);
        }
    }
    __syncthreads();
    double acc[kSvrRows][CPT];
#pragma unroll
    for (int r = 0; r < kSvrRows; ++r)
#pragma unroll
        for (int c = 0; c < CPT; ++c) acc[r][c] = 0.0;

    for (int c = 0; c < nch; ++c) {
        const int st = c % kSvrStages;
        if (tid == 0 && c + kSvrStages - 1 < nch) {          // refill the stage consumed at c - 1
            const int cn = c + kSvrStages - 1, sn = cn % kSvrStages;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_expect_tx(bar + sn, UB + VB);
            bulk_g2s(Ub + (size_t)sn * kSvrJC * kSvrTK, ug + (size_t)cn * kSvrJC * kSvrTK, UB, bar + sn);
            bulk_g2s(Vb + (size_t)sn * kSvrJC * TN, vg + (size_t)cn * kSvrJC * TN, VB, bar + sn);
        }
        mbar_wait(bar + st, (unsigned)((c / kSvrStages) & 1));
        const double* U = Ub + (size_t)st * kSvrJC * kSvrTK + warp * kSvrRows;
        const double* V = Vb + (size_t)st * kSvrJC * TN + lane;
#pragma unroll 4
        for (int jj = 0; jj < kSvrJC; ++jj) {
            double u[kSvrRows];
            const double2* up = reinterpret_cast<const double2*>(U + jj * kSvrTK);
#pragma unroll
            for (int r = 0; r < kSvrRows / 2; ++r) {
                const double2 t = up[r];                    // warp-uniform: broadcast
                u[2 * r] = t.x;
                u[2 * r + 1] = t.y;
            }
#pragma unroll
            for (int cc = 0; cc < CPT; ++cc) {
                const double v = V[jj * TN + cc * 32];
#pragma unroll
                for (int r = 0; r < kSvrRows; ++r) acc[r][cc] = __fma_rn(u[r], v, acc[r][cc]);
            }
        }
        __syncthreads();                                     // stage st free for refill
    }
    // split z writes partial plane z; finish_tile sums the planes in split order
    const size_t plane = (size_t)a.n_k * a.n_f;
    double* P = a.P + (size_t)blockIdx.z * plane;
    const long long kb = a.slab0 + (long long)kt * kSvrTK;
#pragma unroll
    for (int r = 0; r < kSvrRows; ++r) {
        const long long k = kb + warp * kSvrRows + r;
        if (k >= a.slab0 + a.nks) continue;
#pragma unroll
        for (int cc = 0; cc < CPT; ++cc) {
            const int i = it * TN + cc * 32 + lane;
            if (i < a.n_f) P[(size_t)k * a.n_f + i] = acc[r][cc];
        }
    }
}

// One (kernel k, clock i) value of a model: add the SVR member (split partials in split order,
// then the intercept; ensemble order Q7: the SVR member comes last).
__device__ __forceinline__ void add_svr_unit(const DevModel& m, double* r, long long k, long long n_k, int n_f,
                                             int i) {
    const size_t plane = (size_t)n_k * n_f;
    const double* p = m.svr_p + (size_t)k * n_f + i;
    const int Z = m.svr_splits;
    double part[kSvrMaxSplits];                              // all split loads in flight at once
#pragma unroll
    for (int q = 0; q < kSvrMaxSplits; ++q) part[q] = q < Z ? __ldcg(p + q * plane) : 0.0;
    double s = part[0];
#pragma unroll
    for (int q = 1; q < kSvrMaxSplits; ++q)
        if (q < Z) s = __dadd_rn(s, part[q]);
    const double svr = __dadd_rn(s, m.svr_b);
    *r = __dadd_rn(*r, m.svr_weight == 1.0 ? svr : __dmul_rn(m.svr_weight, svr));
}

}  // namespace syn
