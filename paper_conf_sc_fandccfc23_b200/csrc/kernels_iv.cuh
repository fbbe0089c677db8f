// kernels_iv.cuh — clock-interval traversal (CIT) fused sweep kernel for sm_100a.
//
// Same result as k_sweep (bit for bit), far less tree work.  For a fixed kernel k only the
// clock input varies across the n_f evaluations, so each tree is a step function of the clock
// index: static splits are decided once by k's features, a clock split with threshold thr sends
// clocks f_i <= thr left, i.e. cuts the clock-index interval at s = #{i : f_i <= thr} (the table
// is strictly ascending).  One depth-first walk per (kernel, tree) over [0, n_f) visits only the
// nodes some clock reaches (~60 on the bench forests instead of n_f * D = 2352 decisions) and
// emits the runs [lo, hi) of clocks sharing a leaf, in increasing lo.
//
//   phase 1  one (kernel, tree) task per thread: walk_tree -> run starts as a bitmask over the
//            clock axis plus an inclusive popcount prefix per 32-bit word, run values (fp64) in
//            shared memory;
//   phase 2  one (kernel, clock) unit per thread slot: for every tree IN TREE ORDER
//            run = prefix[w] + popc(mask[w] & lanes<=i) - 1; acc += value[run]  (fp64, _rn)
//   finish   linear member, forest mean, default-clock normalisation, per-target argmin
//            (finish_tile, shared with k_sweep).
// Each evaluation still adds the same fp32 leaves (widened to fp64) in the same tree order as
// the oracle, so predictions are identical, not merely close.  A task with more than vcap runs
// keeps its first vcap values; clocks in later runs fall back to a direct root-to-leaf walk.
#pragma once
#include "kernels.cuh"

namespace syn {

constexpr int kMaxStack = 64;   // >= SYNERGY_MAX_DEPTH: pending right parts of ancestors

// Clock cut: s = #{i : f_i <= thr} for fr[lo] <= thr < fr[hi-1].  A uniform grid over the
// clock range gives a start index (grid[b] = #{i : f_i < f_0 + b*step}); the exact position is
// then reached by comparing against the table itself, so the result is exact whatever the
// rounding of b (the grid is only a hint).
__device__ __forceinline__ int clock_cut(const float* fr, const unsigned short* grid, float f0,
                                         float inv_step, float thr, int lo, int hi) {
    int b = __float2int_rz((thr - f0) * inv_step);
    b = min(max(b, 0), kGrid);
    int s = min(max((int)grid[b], lo + 1), hi - 1);
    while (s > lo + 1 && !(fr[s - 1] <= thr)) --s;
    while (s < hi - 1 && fr[s] <= thr) ++s;
    return s;
}

__device__ __forceinline__ int walk_tree(const uint2* __restrict__ nodes, int root,
                                         const float* xrow, int F, const float* fr, int n_f,
                                         const unsigned short* grid, float f0, float inv_step,
                                         uint2* mp, int W, double* vals, int vcap) {
    for (int w = 0; w < W; ++w) mp[w].x = 0u;
    int st_node[kMaxStack];
    int st_iv[kMaxStack];
    int sp = 0, cnt = 0;
    int n = root, lo = 0, hi = n_f;
    while (true) {
        const uint2 nd = ldg_node(nodes + n);
        const int code = (int)(nd.y & 0xffu);
        const float thr = __uint_as_float(nd.x);
        const int child = n + ((int)nd.y >> kCodeBits);
        if (code > F) {                          // leaf: run [lo, hi) takes this value
            if (cnt < vcap) vals[cnt] = (double)thr;
            mp[lo >> 5].x |= 1u << (lo & 31);
            ++cnt;
            if (sp == 0) break;
            --sp;
            n = st_node[sp];
            lo = st_iv[sp] & 0xffff;
            hi = st_iv[sp] >> 16;
            continue;
        }
        bool right;
        if (code < F) {                          // static feature: one side for every clock
            right = !(xrow[code] <= thr);
        } else {
            const bool all_left = fr[hi - 1] <= thr;
            right = !(fr[lo] <= thr);            // whole interval right (NaN thr too)
            if (!all_left && !right) {           // cut: fr[lo] <= thr < fr[hi-1]
                const int s = clock_cut(fr, grid, f0, inv_step, thr, lo, hi);
                st_node[sp] = child + 1;
                st_iv[sp] = s | (hi << 16);
                ++sp;
                hi = s;
            }
        }
        n = child + (right ? 1 : 0);
    }
    int p = 0;
    for (int w = 0; w < W; ++w) {
        mp[w].y = (unsigned)p;
        p += __popc(mp[w].x);
    }
    return cnt;
}

// Root-to-leaf walk for one clock (fallback for runs beyond vcap); xrow[F+1] holds NaN.
__device__ __forceinline__ float direct_leaf(const DevModel& m, int t, const float* xrow, float f, int F) {
    const int2 td = __ldg(m.trees + t);
    int idx = td.x;
    for (int d = 0; d < td.y; ++d) {
        const uint2 n = ldg_node(m.nodes + idx);
        const int code = (int)(n.y & 0xffu);
        const float x = (code == F) ? f : xrow[code];
        idx += ((int)n.y >> kCodeBits) + (x <= __uint_as_float(n.x) ? 0 : 1);
    }
    return __uint_as_float(ldg_node(m.nodes + idx).x);
}

// Model output from its accumulated forest sum (oracle order: linear member first).
__device__ __forceinline__ double combine(const DevModel& m, double acc, const float* xrow, float f, int F) {
    double out = 0.0;
    if (m.lin_weight != 0.0) {
        double lin = m.lin_b;
        for (int j = 0; j < F; ++j) lin = __fma_rn(__ldg(m.lin_w + j), (double)xrow[j], lin);
        lin = __fma_rn(__ldg(m.lin_w + F), (double)f, lin);
        out = __dadd_rn(out, m.lin_weight == 1.0 ? lin : __dmul_rn(m.lin_weight, lin));
    }
    if (m.forest_weight != 0.0) {
        const double forest = __ddiv_rn(acc, (double)m.n_trees);
        out = __dadd_rn(out, m.forest_weight == 1.0 ? forest : __dmul_rn(m.forest_weight, forest));
    }
    return out;
}

template <int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB) k_sweep_iv(const __grid_constant__ SweepArgs a) {
    extern __shared__ __align__(16) unsigned char smem[];
    const int TK = a.tile_k, TC = a.tc, W = a.words, VC = a.vcap, VS = a.vs;
    const long long k0 = (long long)blockIdx.x * TK;
    const int nk = (int)min((long long)TK, a.n_k - k0);
    const int n_f = a.n_f;
    const int F = a.F;
    const int XS = a.xs;
    // layout: acc (2 x TK*n_f doubles) | tasks (mask words, run values) | fr | xk | grid
    double* accS = reinterpret_cast<double*>(smem);
    double* accE = accS + (size_t)TK * n_f;
    uint2* mp = reinterpret_cast<uint2*>(accE + (size_t)TK * n_f);        // [TC*TK][W]
    double* vals = reinterpret_cast<double*>(mp + (size_t)TC * TK * W);   // [TC*TK][VS]
    float* fr = reinterpret_cast<float*>(reinterpret_cast<unsigned char*>(mp) + a.region);
    float* xk = fr + n_f;
    unsigned short* grid = reinterpret_cast<unsigned short*>(xk + TK * XS);

    const float* gfeat = a.features + k0 * F;
    for (int e = threadIdx.x; e < nk * F; e += NT) {
        const int r = e / F;
        xk[r * XS + (e - r * F)] = __ldg(gfeat + e);
    }
    for (int r = threadIdx.x; r < nk; r += NT) {
        xk[r * XS + F] = 0.0f;
        xk[r * XS + F + 1] = CUDART_NAN_F;
    }
    for (int i = threadIdx.x; i < n_f; i += NT) fr[i] = __ldg(a.freqs + i);
    const int units = nk * n_f;
    for (int u = threadIdx.x; u < units; u += NT) { accS[u] = 0.0; accE[u] = 0.0; }
    // clock-cut grid: grid[b] = #{i : f_i < f_0 + b * step}, b = 0..kGrid
    const float f0 = __ldg(a.freqs);
    const float span = __ldg(a.freqs + n_f - 1) - f0;
    const float step = span > 0.0f ? span / (float)kGrid : 1.0f;
    const float inv_step = 1.0f / step;
    for (int b = threadIdx.x; b <= kGrid; b += NT) {
        const float edge = f0 + (float)b * step;
        int l = 0, h = n_f;                          // first index with f_i >= edge
        while (l < h) {
            const int m = (l + h) >> 1;
            if (__ldg(a.freqs + m) < edge) l = m + 1; else h = m;
        }
        grid[b] = (unsigned short)l;
    }
    __syncthreads();

    const int TS = a.ms.forest_weight != 0.0 ? a.ms.n_trees : 0;
    const int TE = a.me.forest_weight != 0.0 ? a.me.n_trees : 0;
    const int TT = TS + TE;   // speedup trees then energy trees
    for (int g0 = 0; g0 < TT; g0 += TC) {
        const int ntc = min(TC, TT - g0);
        {   // phase 1: task (kernel kl, tree g0 + tc), one per thread
            const int tc = threadIdx.x / TK, kl = threadIdx.x - tc * TK;
            if (tc < ntc && kl < nk) {
                const int g = g0 + tc;
                const DevModel& m = g < TS ? a.ms : a.me;
                const int t = g < TS ? g : g - TS;
                const int task = tc * TK + kl;
                walk_tree(m.nodes, __ldg(m.trees + t).x, xk + kl * XS, F, fr, n_f, grid, f0, inv_step,
                          mp + (size_t)task * W, W, vals + (size_t)task * VS, VC);
            }
        }
        __syncthreads();
        // phase 2: each unit adds the chunk's trees in tree order (accumulator in a register
        // for the chunk, in shared memory across chunks)
        const int nS = max(0, min(ntc, TS - g0));    // trees of the chunk that are speedup trees
        for (int u = threadIdx.x; u < units; u += NT) {
            const int kl = u / n_f;
            const int i = u - kl * n_f;
            const int w = i >> 5;
            const unsigned lmask = (2u << (i & 31)) - 1u;
            const uint2* q0 = mp + (size_t)kl * W + w;
            const double* v0 = vals + (size_t)kl * VS;
            const size_t qstep = (size_t)TK * W, vstep = (size_t)TK * VS;
            double acc = accS[u];
            int tc = 0;
            for (int pass = 0; pass < 2; ++pass) {
                const int tend = pass == 0 ? nS : ntc;
                if (pass == 1) { accS[u] = acc; acc = accE[u]; }
#pragma unroll 4
                for (; tc < tend; ++tc) {
                    const uint2 q = q0[tc * qstep];
                    const int run = (int)q.y + __popc(q.x & lmask) - 1;
                    double v;
                    if (run < VC) {
                        v = v0[tc * vstep + run];
                    } else {
                        const int g = g0 + tc;
                        const DevModel& m = g < TS ? a.ms : a.me;
                        v = (double)direct_leaf(m, g < TS ? g : g - TS, xk + kl * XS, fr[i], F);
                    }
                    acc = __dadd_rn(acc, v);
                }
            }
            accE[u] = acc;
        }
        __syncthreads();
    }

    // model outputs, in place: accS/accE become mS/mE; float scratch reuses the task region
    float* sS = reinterpret_cast<float*>(mp);
    float* sE = sS + (size_t)TK * n_f;
    for (int u = threadIdx.x; u < units; u += NT) {
        const int kl = u / n_f;
        const float* xrow = xk + kl * XS;
        const float fi = fr[u - kl * n_f];
        accS[u] = combine(a.ms, accS[u], xrow, fi, F);
        accE[u] = combine(a.me, accE[u], xrow, fi, F);
    }
    __syncthreads();
    finish_tile(a, accS, accE, sS, sE, nk, k0);
}

}  // namespace syn
