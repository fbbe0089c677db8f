// kernels_da.cuh — order-free difference-array sweep (k_sweep_da), the default fused kernel.
//
// Forest mean (Q8): exact sum of the fp32 leaves, rounded once, / T.  Every fp32 leaf
// of a model is an integer multiple of 2^-s (s from the smallest leaf ulp, computed at model
// creation), so v * 2^s is an exact int64 and integer sums are exact in any order; the host only
// enables this kernel when T * max|v| * 2^s < 2^62.  The final (double)sum * 2^-s is then the
// correctly rounded exact sum — the oracle's value — whatever the order of the adds.
//
// Order-freedom removes all buffering.  One CTA owns one kernel (P = (k', f)); its
// threads pull (model, tree) tasks from a CTA counter.  A task walks its tree with restart walks
// on the 2-level block layout (kernels_ws.cuh: walk(lo) follows clock lo's path and keeps the
// smallest left-turn clock threshold thr_min; its run is [lo, #{f_i <= thr_min})), i.e. one walk
// per run of clocks sharing a leaf instead of one per clock.  Runs become updates of a
// per-(kernel, model) difference array over the clock axis:
//     run 0 (lo = 0):  first += v          (per-lane register, block-reduced at the end)
//     run j >= 1:      D[lo_j] += v_j - v_{j-1}   (one int64 shared atomic)
// After all tasks, acc_i = first + sum_{i' <= i} D[i'] = sum over trees of the leaf clock i
// reaches, exactly.  Then forest = (double)acc * 2^-s / T, linear member, default-clock
// normalisation and per-target argmin (finish_tile) as everywhere else.
#pragma once
#include "kernels_ws.cuh"

namespace syn {

__device__ __forceinline__ void atomic_add_s64(long long* p, long long v) {
    atomicAdd(reinterpret_cast<unsigned long long*>(p), (unsigned long long)v);   // two's complement
}

template <int NT>
__global__ void __launch_bounds__(NT, 1024 / NT) k_sweep_da(const __grid_constant__ SweepArgs a) {
    extern __shared__ __align__(16) unsigned char smem[];
    const int n_f = a.n_f, F = a.F, XS = a.xs;
    const long long k = blockIdx.x;
    long long* D = reinterpret_cast<long long*>(smem);                    // [2][n_f + 1]
    double* mS = reinterpret_cast<double*>(D + 2 * (size_t)(n_f + 1));    // [n_f]
    double* mE = mS + n_f;
    float* sS = reinterpret_cast<float*>(mE + n_f);
    float* sE = sS + n_f;
    float* fr = sE + n_f;
    float* xk = fr + n_f;                                                 // [XS]
    unsigned short* grid = reinterpret_cast<unsigned short*>(xk + XS);    // [kGrid + 1]
    int* counter = reinterpret_cast<int*>(grid + ((kGrid + 2) & ~1));

    for (int j = threadIdx.x; j < F; j += NT) xk[j] = __ldg(a.features + k * F + j);
    if (threadIdx.x == 0) {
        xk[F] = 0.0f;
        xk[F + 1] = CUDART_NAN_F;
        *counter = 0;
    }
    for (int i = threadIdx.x; i < n_f; i += NT) fr[i] = __ldg(a.freqs + i);
    for (int b = threadIdx.x; b <= kGrid; b += NT) grid[b] = __ldg(a.grid + b);
    for (int i = threadIdx.x; i < 2 * (n_f + 1); i += NT) D[i] = 0;
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const unsigned lm_lt = lanemask_lt();
    const unsigned xrow_a = su32(xk), fr_a = su32(fr), grid_a = su32(grid);
    const float f0 = a.f0, inv_step = a.inv_step;
    const float f_last = fr[n_f - 1];
    const int TS = a.ms.forest_weight != 0.0 ? a.ms.n_trees : 0;
    const int TE = a.me.forest_weight != 0.0 ? a.me.n_trees : 0;
    const int TT = TS + TE;
    const int BD = max(TS ? a.ms.bdepth : 1, TE ? a.me.bdepth : 1);

    long long firstS = 0, firstE = 0, vprev = 0;
    int task = -1;                      // -1: idle
    bool isE = false;
    const uint4* blocks = a.ms.blocks;
    double scale = 1.0;
    int root = 0, lo = 0;
    float f_lo = 0.0f, tmin = CUDART_INF_F;
    bool exhausted = false;
    while (true) {
        // refill: idle lanes take the next tasks (warp-aggregated counter bump)
        const bool want = task < 0 && !exhausted;
        const unsigned need = __ballot_sync(0xffffffffu, want);
        if (need) {
            int base = 0;
            const int leader = __ffs(need) - 1;
            if (lane == leader) base = atomicAdd(counter, __popc(need));
            base = __shfl_sync(0xffffffffu, base, leader);
            if (want) {
                const int j = base + __popc(need & lm_lt);
                if (j < TT) {
                    task = j;
                    isE = j >= TS;
                    const DevModel& m = isE ? a.me : a.ms;
                    blocks = m.blocks;
                    scale = m.fx_scale;
                    root = __ldg(m.broot + (isE ? j - TS : j));
                    lo = 0;
                    f_lo = lds_f(fr_a);
                    tmin = CUDART_INF_F;
                } else {
                    exhausted = true;
                }
            }
        }
        if (!__any_sync(0xffffffffu, task >= 0)) break;
        // one restart walk per busy lane, lockstep over BD block steps
        float leaf = 0.0f;
        int bk = root;
        bool done = task < 0;
#pragma unroll 2
        for (int d = 0; d < BD; ++d)
            if (!done) block_step(blocks, bk, done, leaf, tmin, f_lo, xrow_a, F);
        if (task >= 0) {
            const int hi = (tmin < f_last) ? clock_cut_s(fr_a, grid_a, f0, inv_step, tmin, lo, n_f) : n_f;
            const long long v = __double2ll_rn(__dmul_rn((double)leaf, scale));   // exact
            if (lo == 0) {
                if (isE) firstE += v; else firstS += v;
            } else {
                atomic_add_s64(D + (isE ? n_f + 1 : 0) + lo, v - vprev);
            }
            vprev = v;
            if (hi >= n_f) {
                task = -1;
            } else {
                lo = hi;
                f_lo = lds_f(fr_a + 4u * (unsigned)hi);
                tmin = CUDART_INF_F;
            }
        }
    }
    // first-run values: warp reduce, one atomic per warp and model
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
        firstS += __shfl_xor_sync(0xffffffffu, firstS, off);
        firstE += __shfl_xor_sync(0xffffffffu, firstE, off);
    }
    if (lane == 0) {
        if (firstS) atomic_add_s64(D, firstS);
        if (firstE) atomic_add_s64(D + n_f + 1, firstE);
    }
    __syncthreads();

    // prefix sums over clocks (warp 0: speedup, warp 1: energy), exact, then model outputs
    const int warp = threadIdx.x >> 5;
    if (warp < 2) {
        const DevModel& m = warp ? a.me : a.ms;
        const long long* Dm = D + (warp ? n_f + 1 : 0);
        double* out = warp ? mE : mS;
        const int chunk = (n_f + 31) / 32;
        const int i0 = min(n_f, lane * chunk), i1 = min(n_f, i0 + chunk);
        long long run = 0;
        for (int i = i0; i < i1; ++i) run += Dm[i];
        long long excl = run;                                 // inclusive scan of chunk sums
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const long long y = __shfl_up_sync(0xffffffffu, excl, off);
            if (lane >= off) excl += y;
        }
        excl -= run;
        const double inv = m.fx_inv;
        for (int i = i0; i < i1; ++i) {
            excl += Dm[i];
            const double forest_sum = __dmul_rn(__ll2double_rn(excl), inv);   // RN(exact sum)
            out[i] = combine(m, forest_sum, xk, fr[i], F);
        }
    }
    __syncthreads();
    finish_tile(a, mS, mE, sS, sE, 1, k);
}

}  // namespace syn
