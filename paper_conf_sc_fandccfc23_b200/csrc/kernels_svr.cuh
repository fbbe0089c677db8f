// kernels_svr.cuh — SVR_RBF member over a clock sweep (Table 2; Q24).
//
// With z = (x - mean) / scale the squared distance of (kernel k, clock f_i) to support vector j
// splits into a static-feature part and a clock part,
//   ||z(k, f_i) - sv_j||^2 = A_kj + B_ji,  A_kj = sum_{d<F} (z_kd - sv_jd)^2,  B_ji = (z(f_i) - sv_jF)^2,
// so svr(k, f_i) = b + sum_j U_kj V_ji with U_kj = dual_j e^{-gamma A_kj}, V_ji = e^{-gamma B_ji}:
// an fp64 [n_k x n_sv] x [n_sv x n_f] contraction.  tcgen05 has no fp64 kind, so it runs on the
// fp64 FMA pipe: each thread holds an 8-kernel x CPT-clock register tile, U is computed in the
// CTA (exp per (k, j) once), V once per call by k_svr_v.  SV ranges are split across CTAs
// (blockIdx.z) when the batch is too small to fill the GPU; finish_tile adds the partials in
// split order.
#pragma once
#include "internal.h"

namespace syn {

// V[j][i] = exp(-gamma * (z(f_i) - sv[j][F])^2)
__global__ void __launch_bounds__(256) k_svr_v(const __grid_constant__ SvrArgs a) {
    const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (long long)a.n_sv * a.n_f) return;
    const int j = (int)(t / a.n_f), i = (int)(t - (long long)j * a.n_f);
    const int F = a.F;
    const double zc = __ddiv_rn(__dsub_rn((double)__ldg(a.freqs + i), __ldg(a.in_mean + F)), __ldg(a.in_scale + F));
    const double b = __dsub_rn(zc, (double)__ldg(a.sv + (size_t)j * (F + 1) + F));
    a.V[t] = exp(-__dmul_rn(a.gamma, __dmul_rn(b, b)));
}

template <int CPT>
__global__ void __launch_bounds__(256, 1) k_svr(const __grid_constant__ SvrArgs a) {
    extern __shared__ __align__(16) double svm[];
    constexpr int TN = 32 * CPT;
    const int F = a.F;
    double* z = svm;                              // [F][kSvrTK] standardized static features
    double* U = z + (size_t)F * kSvrTK;           // [kSvrJC][kSvrTK]
    double* V = U + kSvrJC * kSvrTK;              // [kSvrJC][TN]
    const long long k0 = (long long)blockIdx.x * kSvrTK;
    const int nk = (int)min((long long)kSvrTK, a.n_k - k0);
    const int i0 = blockIdx.y * TN;
    const int j_beg = blockIdx.z * a.sv_per_split;
    const int j_end = min(a.n_sv, j_beg + a.sv_per_split);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

    for (int e = tid; e < kSvrTK * F; e += 256) {
        const int kk = e / F, d = e - kk * F;
        double v = 0.0;
        if (kk < nk)
            v = __ddiv_rn(__dsub_rn((double)__ldg(a.features + k0 * F + e), __ldg(a.in_mean + d)), __ldg(a.in_scale + d));
        z[d * kSvrTK + kk] = v;
    }
    double acc[kSvrRows][CPT];
#pragma unroll
    for (int r = 0; r < kSvrRows; ++r)
#pragma unroll
        for (int c = 0; c < CPT; ++c) acc[r][c] = 0.0;

    for (int j0 = j_beg; j0 < j_end; j0 += kSvrJC) {
        const int jn = min(kSvrJC, j_end - j0);
        __syncthreads();                          // z staged / previous chunk consumed
        for (int u = tid; u < kSvrJC * kSvrTK; u += 256) {
            const int kk = u % kSvrTK, jj = u / kSvrTK;
            double val = 0.0;
            if (jj < jn && kk < nk) {
                const float* s = a.sv + (size_t)(j0 + jj) * (F + 1);
                double A = 0.0;
                for (int d = 0; d < F; ++d) {
                    const double t = __dsub_rn(z[d * kSvrTK + kk], (double)__ldg(s + d));
                    A = __dadd_rn(A, __dmul_rn(t, t));
                }
                val = __dmul_rn(__ldg(a.dual + j0 + jj), exp(-__dmul_rn(a.gamma, A)));
            }
            U[u] = val;
        }
        for (int u = tid; u < kSvrJC * TN; u += 256) {
            const int jj = u / TN, c = u - jj * TN, i = i0 + c;
            V[u] = (jj < jn && i < a.n_f) ? a.V[(size_t)(j0 + jj) * a.n_f + i] : 0.0;
        }
        __syncthreads();
        for (int jj = 0; jj < jn; ++jj) {
            double u[kSvrRows];
            const double2* up = reinterpret_cast<const double2*>(U + jj * kSvrTK + warp * kSvrRows);
#pragma unroll
            for (int r = 0; r < kSvrRows / 2; ++r) {
                const double2 t = up[r];          // warp-uniform: one broadcast wavefront
                u[2 * r] = t.x;
                u[2 * r + 1] = t.y;
            }
#pragma unroll
            for (int c = 0; c < CPT; ++c) {
                const double v = V[jj * TN + c * 32 + lane];
#pragma unroll
                for (int r = 0; r < kSvrRows; ++r) acc[r][c] = __fma_rn(u[r], v, acc[r][c]);
            }
        }
    }
    const size_t plane = (size_t)a.n_k * a.n_f;
    double* P = a.P + (size_t)blockIdx.z * plane;
#pragma unroll
    for (int r = 0; r < kSvrRows; ++r) {
        const int kk = warp * kSvrRows + r;
        if (kk >= nk) continue;
#pragma unroll
        for (int c = 0; c < CPT; ++c) {
            const int i = i0 + c * 32 + lane;
            if (i < a.n_f) P[(size_t)(k0 + kk) * a.n_f + i] = acc[r][c];
        }
    }
}

// Model row kl of kernel k: add the SVR member (partials in split order, then the intercept).
__device__ __forceinline__ void add_svr_row(const DevModel& m, double* r, long long k, long long n_k, int n_f,
                                            int lane) {
    if (m.svr_weight == 0.0) return;
    const size_t plane = (size_t)n_k * n_f;
    const double* p = m.svr_p + (size_t)k * n_f;
    for (int i = lane; i < n_f; i += 32) {
        double s = p[i];
        for (int q = 1; q < m.svr_splits; ++q) s = __dadd_rn(s, p[q * plane + i]);
        const double svr = __dadd_rn(s, m.svr_b);
        r[i] = __dadd_rn(r[i], m.svr_weight == 1.0 ? svr : __dmul_rn(m.svr_weight, svr));
    }
    __syncwarp();
}

}  // namespace syn
