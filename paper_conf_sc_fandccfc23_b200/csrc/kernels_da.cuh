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
// The kernel is bound by the L1 wavefront rate of the scattered block loads and lives on L1 hits of
// the upper tree blocks, which every restart walk re-reads; shared memory is kept small so L1 stays
// large.  Optional TOPC (SYNERGY_TOPC=1) instead stages each task's top two block levels (root + 4
// grandchild blocks, 160 B per thread) in shared memory: measured slower on B200 (round 1) because
// the extra 20 KB per CTA comes out of L1.
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

// Model m of the call: 0 speedup, 1 energy, 2 direct EDP, 3 direct ED2P (four-model variant).
__device__ __forceinline__ const DevModel& da_model(const SweepArgs& a, int m) {
    return m == 0 ? a.ms : m == 1 ? a.me : a.mx[m - 2];
}

__device__ __forceinline__ int da_trees(const SweepArgs& a, int m) {
    if (m >= 2 && !a.has_x[m - 2]) return 0;
    const DevModel& d = da_model(a, m);
    return d.forest_weight != 0.0 ? d.n_trees : 0;
}

template <int NT, bool TOPC>
__global__ void __launch_bounds__(NT, 1024 / NT) k_sweep_da(const __grid_constant__ SweepArgs a) {
    extern __shared__ __align__(16) unsigned char smem[];
    const int n_f = a.n_f, F = a.F, XS = a.xs, KPC = a.tile_k;
    const int NM = (a.has_x[0] || a.has_x[1]) ? 4 : 2;                      // models in this call
    const long long k0 = (long long)blockIdx.x * KPC;
    const int nk = (int)min((long long)KPC, a.n_k - k0);
    long long* D = reinterpret_cast<long long*>(smem);                      // [KPC][NM][n_f + 1]
    long long* first = D + (size_t)KPC * NM * (n_f + 1);                   // [NT][KPC][NM]
    double* mv0 = reinterpret_cast<double*>(first + (size_t)NT * KPC * NM); // [NM][KPC][n_f]
    float* sv0 = reinterpret_cast<float*>(mv0 + (size_t)NM * KPC * n_f);    // [NM][KPC][n_f]
    float* fr = sv0 + (size_t)NM * KPC * n_f;
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
    for (int i = threadIdx.x; i < KPC * NM * (n_f + 1); i += NT) D[i] = 0;
    long long* myfirst = first + (size_t)threadIdx.x * KPC * NM;
    for (int i = 0; i < KPC * NM; ++i) myfirst[i] = 0;
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const unsigned lm_lt = lanemask_lt();
    const unsigned xk_a = su32(xk), fr_a = su32(fr), grid_a = su32(grid);
    const unsigned topc_a = su32(topc) + (unsigned)threadIdx.x * 160u;
    const float f0 = a.f0, inv_step = a.inv_step;
    const float f_last = fr[n_f - 1];
    // tasks of one kernel: the trees of model 0, then 1, 2, 3 (cumulative counts c1 < c2 < c3 < TT)
    const int T0 = da_trees(a, 0), T1 = da_trees(a, 1), T2 = NM > 2 ? da_trees(a, 2) : 0,
              T3 = NM > 2 ? da_trees(a, 3) : 0;
    const int c1 = T0, c2 = c1 + T1, c3 = c2 + T2, TT = c3 + T3;
    // a task is (kernel, model, tree, clock sub-range r of R): small batches split each tree's
    // clock axis so more lanes share the walks (order-free sums make the pieces independent)
    const int R = max(1, a.nsub);
    const int n_tasks = nk * TT * R;
    int BD = 1;
    for (int m = 0; m < NM; ++m)
        if (da_trees(a, m)) BD = max(BD, da_model(a, m).bdepth);

    long long vprev = 0;
    int task = -1;                      // -1: idle
    int kl = 0, mi = 0, ra = 0, rb = n_f;   // sub-range [ra, rb) of the clock axis
    double scale = 1.0;
    int root = 0, lo = 0;
    const uint4* own = a.ms.blocks;
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
                    kl = j / (TT * R);
                    const int rem = j - kl * TT * R;
                    const int jj = rem / R, r = rem - jj * R;
                    ra = (int)(((long long)r * n_f) / R);
                    rb = (int)(((long long)(r + 1) * n_f) / R);
                    mi = jj < c1 ? 0 : jj < c2 ? 1 : jj < c3 ? 2 : 3;
                    const int tree = jj - (mi == 0 ? 0 : mi == 1 ? c1 : mi == 2 ? c2 : c3);
                    const DevModel& m = da_model(a, mi);
                    scale = m.fx_scale;
                    own = m.blocks;
                    root = __ldg(m.broot + tree);
                    xrow_a = xk_a + 4u * (unsigned)(kl * XS);
                    if (TOPC) {                               // stage the top two block levels
                        const uint4 A0 = ldg_blk(own + 2 * (size_t)root), B0 = ldg_blk(own + 2 * (size_t)root + 1);
                        sts_blk(topc_a, A0);
                        sts_blk(topc_a + 16u, B0);
                        const unsigned cw = A0.w;
                        const unsigned gs[4] = {B0.x, B0.y, B0.z, B0.w};
#pragma unroll
                        for (int s2 = 0; s2 < 4; ++s2) {
                            const bool inner = (int)(cw & 0xffu) <= F && (int)((cw >> (8 + 8 * (s2 >> 1))) & 0xffu) <= F &&
                                               !((cw >> (24 + s2)) & 1u);
                            if (inner) {
                                sts_blk(topc_a + 32u * (1 + s2), ldg_blk(own + 2 * (size_t)gs[s2]));
                                sts_blk(topc_a + 32u * (1 + s2) + 16u, ldg_blk(own + 2 * (size_t)gs[s2] + 1));
                            }
                        }
                    }
                    lo = ra;
                    f_lo = lds_f(fr_a + 4u * (unsigned)min(ra, n_f - 1));
                    tmin = CUDART_INF_F;
                    if (ra >= rb) task = -1;                  // empty sub-range (R > n_f)
                } else {
                    exhausted = true;
                }
            }
        }
        if (!__any_sync(0xffffffffu, task >= 0)) break;
        // one restart walk per busy lane, lockstep over BD 2-level block steps
        float leaf = 0.0f;
        int bk = root;
        bool done = task < 0;
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
            long long* Drow = D + ((size_t)kl * NM + mi) * (n_f + 1);
            if (lo == 0) myfirst[kl * NM + mi] += v;                               // thread-private
            else atomic_add_s64(Drow + lo, lo == ra ? v : v - vprev);             // sub-range start: +v
            vprev = v;
            if (hi >= rb) {                                                        // run reaches the range end
                if (rb < n_f) atomic_add_s64(Drow + rb, -v);
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
    for (int p = warp; p < NM * nk; p += nw) {            // p = kernel * NM + model
        const int pk = p / NM, pm = p - pk * NM;
        if (pm >= 2 && !a.has_x[pm - 2]) continue;
        long long s = 0;
        for (int t2 = lane; t2 < NT; t2 += 32) s += first[(size_t)t2 * KPC * NM + p];
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
        long long* Dm = D + (size_t)p * (n_f + 1);
        if (lane == 0) Dm[0] += s;
        __syncwarp();
        const DevModel& m = da_model(a, pm);
        double* out = mv0 + ((size_t)pm * KPC + pk) * n_f;
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
    double* mv[4];
    float* sv[4];
    for (int m = 0; m < 4; ++m) {
        const bool present = m < 2 || (NM > 2 && a.has_x[m - 2]);
        mv[m] = present ? mv0 + (size_t)m * KPC * n_f : nullptr;
        sv[m] = present ? sv0 + (size_t)m * KPC * n_f : nullptr;
    }
    finish_tile4(a, mv, sv, nk, k0);
}

}  // namespace syn
