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
// Block loads are lane-paired: lanes 2i and 2i+1 fetch the two 16-byte halves of the SAME 32-byte
// block in one instruction (one L1 sector for two lanes, the L1 wavefront rate being the bound of
// this kernel), then trade the one grandchild word each needs with a shuffle.
#pragma once
#include "kernels_ws.cuh"

namespace syn {

__device__ __forceinline__ void atomic_add_s64(long long* p, long long v) {
    atomicAdd(reinterpret_cast<unsigned long long*>(p), (unsigned long long)v);   // two's complement
}

// Clock cut with the hint grid read through L1 (built once per clock table, syn_clocks).
__device__ __forceinline__ int clock_cut_g(unsigned fr_a, const unsigned short* __restrict__ grid,
                                           float f0, float inv_step, float thr, int lo, int hi) {
    int b = __float2int_rz((thr - f0) * inv_step);
    b = min(max(b, 0), kGrid);
    int s = min(max((int)__ldg(grid + b), lo + 1), hi - 1);
    while (s > lo + 1 && !(lds_f(fr_a + 4u * (s - 1)) <= thr)) --s;
    while (s < hi - 1 && lds_f(fr_a + 4u * s) <= thr) ++s;
    return s;
}

// One lane-paired 2-level block step, executed by all 32 lanes (warp-synchronous).  Lane state:
// bk = block index in its own model's array, isE = model, done = no walk / walk finished.
__device__ __forceinline__ void pair_block_step(const uint4* __restrict__ bS, const uint4* __restrict__ bE,
                                                int& bk, bool isE, bool& done, float& leaf, float& tmin,
                                                float f, unsigned xrow_a, int F, bool odd) {
    const int info = done ? -1 : ((bk << 1) | (isE ? 1 : 0));
    const int pinfo = __shfl_xor_sync(0xffffffffu, info, 1);
    const int xinfo = odd ? pinfo : info;            // the even lane's block
    const int yinfo = odd ? info : pinfo;            // the odd lane's block
    uint4 r1 = make_uint4(0u, 0u, 0u, 0u), r2 = make_uint4(0u, 0u, 0u, 0u);
    if (xinfo >= 0) r1 = ldg_blk(((xinfo & 1) ? bE : bS) + 2 * (size_t)(xinfo >> 1) + (odd ? 1 : 0));
    if (yinfo >= 0) r2 = ldg_blk(((yinfo & 1) ? bE : bS) + 2 * (size_t)(yinfo >> 1) + (odd ? 0 : 1));
    const uint4 A = odd ? r2 : r1;                   // own block, words 0..3
    const uint4 Bp = odd ? r1 : r2;                  // partner's block, words 4..7
    int slot = 0;
    bool need = false;
    if (!done) {
        const unsigned codes = A.w;
        const int cn = (int)(codes & 0xffu);
        const float tn = __uint_as_float(A.x);
        if (cn > F) {                                // one-leaf tree
            leaf = tn;
            done = true;
        } else {
            const float xn = (cn == F) ? f : lds_f(xrow_a + 4u * (unsigned)cn);
            const bool r0 = !(xn <= tn);
            if (cn == F && !r0) tmin = fminf(tmin, tn);
            const float tc = __uint_as_float(r0 ? A.z : A.y);
            const int cc = (int)((codes >> (r0 ? 16 : 8)) & 0xffu);
            if (cc > F) {                            // child leaf (odd depth)
                leaf = tc;
                done = true;
            } else {
                const float xc = (cc == F) ? f : lds_f(xrow_a + 4u * (unsigned)cc);
                const bool r1b = !(xc <= tc);
                if (cc == F && !r1b) tmin = fminf(tmin, tc);
                slot = (r0 ? 2 : 0) + (r1b ? 1 : 0);
                need = true;
                if ((codes >> (24 + slot)) & 1u) done = true;   // grandchild is a leaf
            }
        }
    }
    const int pslot = __shfl_xor_sync(0xffffffffu, slot, 1);
    const unsigned give = pslot == 0 ? Bp.x : pslot == 1 ? Bp.y : pslot == 2 ? Bp.z : Bp.w;
    const unsigned g = __shfl_xor_sync(0xffffffffu, give, 1);
    if (need) {
        if (done) leaf = __uint_as_float(g);
        else bk = (int)g;
    }
}

template <int NT, bool PAIR>
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
    const bool odd = lane & 1;
    const unsigned lm_lt = lanemask_lt();
    const unsigned xk_a = su32(xk), fr_a = su32(fr), grid_a = su32(grid);
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
        if (PAIR) {
            for (int d = 0; d < BD; ++d)
                pair_block_step(bS, bE, bk, isE, done, leaf, tmin, f_lo, xrow_a, F, odd);
        } else {
            const uint4* __restrict__ own = isE ? bE : bS;
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
