// kernels_da.cuh — order-free difference-array sweep (k_sweep_da), the default fused kernel.
//
// Forest mean (Q8): exact sum of the fp32 leaves, rounded once, / T.  Every fp32 leaf
// of a model is an integer multiple of 2^-s (s from the smallest leaf ulp, computed at model
// creation), so v * 2^s is an exact int64 and integer sums are exact in any order; the host only
// enables this kernel when T * max|v| * 2^s < 2^62.  The final (double)sum * 2^-s is then the
// correctly rounded exact sum — the oracle's value — whatever the order of the adds.
//
// Order-freedom removes all buffering.  A CTA owns KPC kernels (P = (k', f)); its
// threads pull (kernel, model, tree) tasks from a CTA counter.  A task walks its tree with
// restart walks on the 2-level block layout: walk(lo) follows clock lo's path and keeps the
// smallest left-turn clock threshold thr_min; its run is [lo, #{f_i <= thr_min}) (kernels_ws.cuh),
// i.e. one walk per run of clocks sharing a leaf instead of one per clock.  Runs become updates of
// a per-(kernel, model) difference array over the clock axis:
//     run 0 (lo = 0):  first[thread][kernel][model] += v      (thread-private, no atomic)
//     run j >= 1:      D[kernel][model][lo_j] += v_j - v_{j-1}  (one int64 shared atomic)
// After all tasks, acc_i = sum(first) + sum_{i' <= i} D[i'] = sum over trees of the leaf clock i
// reaches, exactly.  Then forest = (double)acc * 2^-s / T, linear member, default-clock
// normalisation and per-target argmin (finish_tile) as everywhere else.
//
// The kernel is bound by the L1 wavefront rate of the scattered block loads.  Every restart walk
// of a task re-traverses the top of the same tree, so at task start each thread stages the root
// block and its four grandchild blocks (the top two block levels, 160 B) in shared memory and the
// walks read levels 0-1 from there (TOPC; about a quarter fewer global block loads per task).
#pragma once
#include "kernels_ws.cuh"

namespace syn {

__device__ __forceinline__ void atomic_add_s64(long long* p, long long v) {
    atomicAdd(reinterpret_cast<unsigned long long*>(p), (unsigned long long)v);   // two's complement
}

__device__ __forceinline__ void sts_blk(unsigned a, uint4 v) {
    asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" :: "r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w));
}
__device__ __forceinline__ uint4 lds_blk(unsigned a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}

template <int NT, bool TOPC>
__global__ void __launch_bounds__(NT, 1024 / NT) k_sweep_da(const __grid_constant__ SweepArgs a) {
    extern __shared__ __align__(16) unsigned char smem[];
    const int n_f = a.n_f, F = a.F, XS = a.xs, KPC = a.tile_k;
    const long long k0 = (long long)blockIdx.x * KPC;
    const int nk = (int)min((long long)KPC, a.n_k - k0);
    long long* D = reinterpret_cast<long long*>(smem);                      // [KPC][2][n_f + 1]
    long long* first = D + (size_t)KPC * 2 * (n_f + 1);                    // [NT][KPC][2]
    double* mS = reinterpret_cast<double*>(first + (size_t)NT * KPC * 2);   // [KPC][n_f]
    double* mE = mS + (size_t)KPC * n_f;
    float* sS = reinterpret_cast<float*>(mE + (size_t)KPC * n_f);
    float* sE = sS + (size_t)KPC * n_f;
    float* fr = sE + (size_t)KPC * n_f;
    float* xk = fr + n_f;                                                   // [KPC][XS]
    unsigned short* grid = reinterpret_cast<unsigned short*>(xk + KPC * XS);   // [kGrid + 2]
    int* counter = reinterpret_cast<int*>(grid + kGrid + 2);
    // per-thread cache of its task's top two block levels: root + 4 grandchild blocks (5 x 32 B)
    uint4* topc = reinterpret_cast<uint4*>(smem + a.head_bytes);

    const float* gfeat = a.features + k0 * F;
    for (int e = threadIdx.x; e < nk * F; e += NT) {
        const int r = e / F;
        xk[r * XS + (e - r * F)] = __ldg(gfeat + e);
    }
    for (int r = threadIdx.x; r < KPC; r += NT) {
        xk[r * XS + F] = 0.0f;
        xk[r * XS + F + 1] = CUDART_NAN_F;
    }
    if (threadIdx.x == 0) *counter = 0;
    for (int i = threadIdx.x; i < n_f; i += NT) fr[i] = __ldg(a.freqs + i);
    for (int b = threadIdx.x; b <= kGrid; b += NT) grid[b] = __ldg(a.grid + b);
    for (int i = threadIdx.x; i < KPC * 2 * (n_f + 1); i += NT) D[i] = 0;
    long long* myfirst = first + (size_t)threadIdx.x * KPC * 2;
    for (int i = 0; i < KPC * 2; ++i) myfirst[i] = 0;
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const unsigned lm_lt = lanemask_lt();
    const unsigned xk_a = su32(xk), fr_a = su32(fr), grid_a = su32(grid);
    const unsigned topc_a = su32(topc) + (unsigned)threadIdx.x * 160u;
    const float f0 = a.f0, inv_step = a.inv_step;
    const float f_last = fr[n_f - 1];
    const int TS = a.ms.forest_weight != 0.0 ? a.ms.n_trees : 0;
    const int TE = a.me.forest_weight != 0.0 ? a.me.n_trees : 0;
    const int TT = TS + TE;
    const int n_tasks = nk * TT;
    const int BD = max(TS ? a.ms.bdepth : 1, TE ? a.me.bdepth : 1);
    const uint4* __restrict__ bS = a.ms.blocks;
    const uint4* __restrict__ bE = a.me.blocks;

    long long vprev = 0;
    int task = -1;                      // -1: idle
    int kl = 0;
    bool isE = false;
    double scale = 1.0;
    int root = 0, lo = 0;
    unsigned xrow_a = xk_a;
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
                if (j < n_tasks) {
                    task = j;
                    kl = j / TT;
                    const int jj = j - kl * TT;
                    isE = jj >= TS;
                    const DevModel& m = isE ? a.me : a.ms;
                    scale = m.fx_scale;
                    root = __ldg(m.broot + (isE ? jj - TS : jj));
                    xrow_a = xk_a + 4u * (unsigned)(kl * XS);
                    if (TOPC) {                               // stage the top two block levels
                        const uint4* bl = isE ? bE : bS;
                        const uint4 A0 = ldg_blk(bl + 2 * (size_t)root), B0 = ldg_blk(bl + 2 * (size_t)root + 1);
                        sts_blk(topc_a, A0);
                        sts_blk(topc_a + 16u, B0);
                        const unsigned cw = A0.w;
                        const unsigned gs[4] = {B0.x, B0.y, B0.z, B0.w};
#pragma unroll
                        for (int s2 = 0; s2 < 4; ++s2) {
                            const bool inner = (int)(cw & 0xffu) <= F && (int)((cw >> (8 + 8 * (s2 >> 1))) & 0xffu) <= F &&
                                               !((cw >> (24 + s2)) & 1u);
                            if (inner) {
                                sts_blk(topc_a + 32u * (1 + s2), ldg_blk(bl + 2 * (size_t)gs[s2]));
                                sts_blk(topc_a + 32u * (1 + s2) + 16u, ldg_blk(bl + 2 * (size_t)gs[s2] + 1));
                            }
                        }
                    }
                    lo = 0;
                    f_lo = lds_f(fr_a);
                    tmin = CUDART_INF_F;
                } else {
                    exhausted = true;
                }
            }
        }
        if (!__any_sync(0xffffffffu, task >= 0)) break;
        // one restart walk per busy lane, lockstep over BD lane-paired block steps
        float leaf = 0.0f;
        int bk = root;
        bool done = task < 0;
        const uint4* __restrict__ own = isE ? bE : bS;
        if (TOPC) {                                   // levels 0-1 from the shared cache
            int gs = 0;
            if (!done) block_decide(lds_blk(topc_a), lds_blk(topc_a + 16u), bk, gs, done, leaf, tmin, f_lo, xrow_a, F);
            if (BD > 1 && !done) {
                const unsigned ca = topc_a + 32u * (1 + gs);
                block_decide(lds_blk(ca), lds_blk(ca + 16u), bk, gs, done, leaf, tmin, f_lo, xrow_a, F);
            }
#pragma unroll 2
            for (int d = 2; d < BD; ++d)
                if (!done) block_step(own, bk, done, leaf, tmin, f_lo, xrow_a, F);
        } else {
#pragma unroll 2
            for (int d = 0; d < BD; ++d)
                if (!done) block_step(own, bk, done, leaf, tmin, f_lo, xrow_a, F);
        }
        if (task >= 0) {
            const int hi = (tmin < f_last) ? clock_cut_s(fr_a, grid_a, f0, inv_step, tmin, lo, n_f) : n_f;
            const long long v = __double2ll_rn(__dmul_rn((double)leaf, scale));   // exact
            if (lo == 0) myfirst[kl * 2 + (isE ? 1 : 0)] += v;                    // thread-private
            else atomic_add_s64(D + ((size_t)kl * 2 + (isE ? 1 : 0)) * (n_f + 1) + lo, v - vprev);
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
    __syncthreads();

    // fold the thread-private first-run sums into D[.][.][0], then prefix sums over clocks
    const int warp = threadIdx.x >> 5, nw = NT / 32;
    for (int p = warp; p < 2 * nk; p += nw) {            // p = kernel * 2 + model
        long long s = 0;
        for (int t2 = lane; t2 < NT; t2 += 32) s += first[(size_t)t2 * KPC * 2 + p];
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
        long long* Dm = D + (size_t)p * (n_f + 1);
        if (lane == 0) Dm[0] += s;
        __syncwarp();
        const int pk = p >> 1, pm = p & 1;
        const DevModel& m = pm ? a.me : a.ms;
        double* out = (pm ? mE : mS) + (size_t)pk * n_f;
        const float* xrow = xk + pk * XS;
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
            out[i] = combine(m, forest_sum, xrow, fr[i], F);
        }
    }
    __syncthreads();
    finish_tile(a, mS, mE, sS, sE, nk, k0);
}

}  // namespace syn
