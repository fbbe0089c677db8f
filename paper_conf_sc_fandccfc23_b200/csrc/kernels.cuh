// kernels.cuh — shared finish / selection kernels of the SYnergy predict+select hot path (sm_100a).
//
//   combine()        a model's raw output from its exact forest sum: linear member, forest mean
//                    (Q7/Q8)
//   finish_tile4()   SVR member, default-clock normalisation (L69), then per target the objective /
//                    constraint and the masked lowest-index argmin (L253-L271, L322) on integer
//                    keys with warp min-reductions; used by k_tm_finish and k_gen_finish
//   k_select         standalone selection over predictions in HBM (one warp per kernel)
//   k_pareto, k_choice_error, k_error_reduce, k_plan   NEXT f3 / f4 (Pareto front, choice error,
//                    plan emission)
//
// Arithmetic contract (Q15): the oracle's op sequence — fp64 fma chain for the linear
// member, exact leaf sum rounded once then / T, fp64 normalisation rounded once to fp32, fp64
// thresholds (compared exactly on the floats, see select_target); every fp64 op is an explicit _rn intrinsic and the library is built with
// --fmad=false, so nothing is contracted.  Ties: lexicographic (key, index) minimum.
#pragma once
#include "device_util.cuh"
#include "kernels_svr.cuh"

namespace syn {

__device__ __forceinline__ bool valid_pred(float s, float e) {
    // DESIGN.md Q16: finite and strictly positive speedup and energy
    return isfinite(s) && isfinite(e) && s > 0.0f && e > 0.0f;
}

// Model output from its forest sum (the exact leaf sum rounded once to fp64; oracle order: linear
// member first, then the forest mean; a weight of exactly 1 skips its multiplication, Q7).  The
// linear member's fma chain runs over the F static inputs, then the clock (input F): its static
// part is the same for every clock of a kernel, so linear_static() computes it once per (kernel,
// model) and combine_pre() finishes each clock with the same operations in the same order.
__device__ __forceinline__ double linear_static(const DevModel& m, const float* xrow, int F) {
    double lin = m.lin_b;
    if (m.lin_weight != 0.0)
        for (int j = 0; j < F; ++j) lin = __fma_rn(__ldg(m.lin_w + j), (double)xrow[j], lin);
    return lin;
}
__device__ __forceinline__ double combine_pre(const DevModel& m, double forest_sum, double lin_s, float f, int F) {
    double out = 0.0;
    if (m.lin_weight != 0.0) {
        const double lin = __fma_rn(__ldg(m.lin_w + F), (double)f, lin_s);
        out = __dadd_rn(out, m.lin_weight == 1.0 ? lin : __dmul_rn(m.lin_weight, lin));
    }
    if (m.forest_weight != 0.0) {
        const double forest = __ddiv_rn(forest_sum, (double)m.n_trees);
        out = __dadd_rn(out, m.forest_weight == 1.0 ? forest : __dmul_rn(m.forest_weight, forest));
    }
    return out;
}
__device__ __forceinline__ double combine(const DevModel& m, double forest_sum, const float* xrow, float f, int F) {
    return combine_pre(m, forest_sum, linear_static(m, xrow, F), f, F);
}

// Selection on integer keys.  A valid prediction (Q16) is a positive finite float, and the bit
// patterns of positive finite floats and doubles order like their values; every key below is
// such a value or (MAX_PERF, ES) the complement of one.  So a target's masked lexicographic
// (key, index) minimum is a lane-local strict-< scan in clock order followed by warp
// min-reductions (REDUX): first over the key words, then over the indices of the lanes that hold
// the minimum.  An invalid or infeasible clock has the all-ones key, which no valid key reaches.
__device__ __forceinline__ bool valid_bits(unsigned b) { return b - 1u < 0x7f7fffffu; }   // (0, FLT_MAX]

__device__ __forceinline__ int warp_argmin32(unsigned key, unsigned idx) {
    const unsigned m = __reduce_min_sync(0xffffffffu, key);
    const unsigned i = __reduce_min_sync(0xffffffffu, key == m ? idx : 0xffffffffu);
    return m == 0xffffffffu ? -1 : (int)i;
}

__device__ __forceinline__ int warp_argmin64(unsigned long long key, unsigned idx) {
    const unsigned hi = (unsigned)(key >> 32), lo = (unsigned)key;
    const unsigned mh = __reduce_min_sync(0xffffffffu, hi);
    const unsigned ml = __reduce_min_sync(0xffffffffu, hi == mh ? lo : 0xffffffffu);
    const unsigned i = __reduce_min_sync(0xffffffffu, (hi == mh && lo == ml) ? idx : 0xffffffffu);
    return (mh == 0xffffffffu && ml == 0xffffffffu) ? -1 : (int)i;
}

struct RowBase {
    double E_def, S_def, E_min, S_minE;
};

// Selection baselines of one row (Q14-Q16): false if the default clock's prediction is
// invalid (every target then -1); else E_def, S_def and the minimum-energy point's E_min, S_minE
// (lowest index among equal minima, L265).  Whole warp, result in every lane.
__device__ __forceinline__ bool select_baseline(const float* S, const float* E, int n_f, int def, int lane,
                                                RowBase& b) {
    const float sd = S[def], ed = E[def];
    if (!(valid_bits(__float_as_uint(sd)) && valid_bits(__float_as_uint(ed)))) return false;
    unsigned bk = 0xffffffffu, bi = 0xffffffffu;
    for (int i = lane; i < n_f; i += 32) {
        const unsigned su = __float_as_uint(S[i]), eu = __float_as_uint(E[i]);
        const unsigned k = (valid_bits(su) && valid_bits(eu)) ? eu : 0xffffffffu;
        if (k < bk) { bk = k; bi = i; }
    }
    const int im = warp_argmin32(bk, bi);                          // >= 0: the default is valid
    b.E_def = (double)ed;
    b.S_def = (double)sd;
    b.E_min = (double)E[im];
    b.S_minE = (double)S[im];
    return true;
}

// One target of one row: the lowest index minimising the target's key
// among valid feasible clocks, -1 if none.  frac = x / 100 in fp64 (host-computed, the oracle's
// division).  P2/P3: direct EDP / ED2P predictions or null.  A constraint (double)e <= thr holds
// for a float e iff e <= RD_float(thr) (the largest float not above thr), and (double)s >= thr
// iff s >= RU_float(thr), so the feasibility tests run on the floats.
__device__ __forceinline__ int select_target(const float* S, const float* E, const float* P2, const float* P3,
                                             int n_f, int kd, double frac, const RowBase& b, int lane) {
    if (kd == 2 || kd == 3) {                                       // MIN_EDP e*t, MIN_ED2P e*t^2
        const float* P = kd == 2 ? P2 : P3;
        unsigned long long bk = ~0ull;
        unsigned bi = 0xffffffffu;
        for (int i = lane; i < n_f; i += 32) {
            const float sf = S[i], ef = E[i];
            if (!(valid_bits(__float_as_uint(sf)) && valid_bits(__float_as_uint(ef)))) continue;
            unsigned long long k;
            if (P) {                                                // direct prediction, valid too
                const unsigned pu = __float_as_uint(P[i]);
                if (!valid_bits(pu)) continue;
                k = pu;
            } else {                                                // e / s (/ s): positive finite
                double q = __ddiv_rn((double)ef, (double)sf);
                if (kd == 3) q = __ddiv_rn(q, (double)sf);
                k = (unsigned long long)__double_as_longlong(q);
            }
            if (k < bk) { bk = k; bi = i; }
        }
        return warp_argmin64(bk, bi);
    }
    float ebound = CUDART_INF_F, sbound = -CUDART_INF_F;            // feasible: e <= ebound, s >= sbound
    if (kd == 4)                                                    // ES_x: E <= E_def - x% (E_def - E_min)
        ebound = __double2float_rd(__dsub_rn(b.E_def, __dmul_rn(frac, __dsub_rn(b.E_def, b.E_min))));
    else if (kd == 5)                                               // PL_x: S >= S_def - x% (S_def - S_minE)
        sbound = __double2float_ru(__dsub_rn(b.S_def, __dmul_rn(frac, __dsub_rn(b.S_def, b.S_minE))));
    else if (kd == 6)                                               // ES_ABS_x (L11/L46, Q1): E <= (1 - x%) E_def
        ebound = __double2float_rd(__dmul_rn(__dsub_rn(1.0, frac), b.E_def));
    else if (kd == 7)                                               // PL_ABS_x: S >= (1 - x%) S_def
        sbound = __double2float_ru(__dmul_rn(__dsub_rn(1.0, frac), b.S_def));
    const bool max_s = kd == 0 || kd == 4 || kd == 6;               // key -s: complement of s's bits
    unsigned bk = 0xffffffffu, bi = 0xffffffffu;
    for (int i = lane; i < n_f; i += 32) {
        const float sf = S[i], ef = E[i];
        const unsigned su = __float_as_uint(sf), eu = __float_as_uint(ef);
        const bool ok = valid_bits(su) && valid_bits(eu) && ef <= ebound && sf >= sbound;
        const unsigned k = ok ? (max_s ? ~su : eu) : 0xffffffffu;
        if (k < bk) { bk = k; bi = i; }
    }
    return warp_argmin32(bk, bi);
}

// Every target of one row, one warp (standalone selection and the choice-error truth).
__device__ __forceinline__ void select_row_warp(const float* S, const float* E, const float* P2,
                                                const float* P3, int n_f, int def,
                                                int n_t, const int* kind, const double* frac,
                                                int* out, int lane) {
    RowBase b;
    if (!select_baseline(S, E, n_f, def, lane, b)) {
        for (int t = lane; t < n_t; t += 32) out[t] = -1;
        return;
    }
    for (int t = 0; t < n_t; ++t) {
        const int c = select_target(S, E, P2, P3, n_f, kind[t], frac[t], b, lane);
        if (lane == 0) out[t] = c;
    }
}

// Finish of a tile of nk kernels (all threads of the CTA; caller has synchronised the block).
// mv[m] ([nk][n_f] fp64 raw outputs in shared memory) for models m < 4 — speedup, energy,
// direct EDP, direct ED2P; mv[m] null when absent — and sv[m] the matching float scratch.
//   1. SVR members (add_svr_row's arithmetic), every (row, clock) in parallel
//   2. normalise to the default clock (S = (float)(m_i / m_def), L69 / DESIGN.md Q13; raw
//      (float)m when def == -1), write the predictions if requested
//   3. per (row, target) one warp: baselines + the target's argmin; direct EDP / ED2P
//      predictions become the MIN_EDP / MIN_ED2P keys
__device__ __forceinline__ void finish_tile4(const SweepArgs& a, double* const* mv, float* const* sv,
                                             int nk, long long k0) {
    const int n_f = a.n_f;
    const int lane = threadIdx.x & 31;
    const int nw = blockDim.x >> 5;
    const int units = nk * n_f;
    bool any_svr = false;
    for (int m = 0; m < 4; ++m) {
        if (!mv[m]) continue;
        const DevModel& md = m == 0 ? a.ms : m == 1 ? a.me : a.mx[m - 2];
        if (md.svr_weight == 0.0) continue;
        any_svr = true;
        for (int u = threadIdx.x; u < units; u += blockDim.x) {
            const int kl = u / n_f;
            add_svr_unit(md, mv[m] + u, k0 + kl, a.n_k, n_f, u - kl * n_f);
        }
    }
    if (any_svr) __syncthreads();
    for (int m = 0; m < 4; ++m) {
        if (!mv[m]) continue;
        float* g = m == 0 ? a.S_out : m == 1 ? a.E_out : a.X_out[m - 2];
#pragma unroll 4
        for (int u = threadIdx.x; u < units; u += blockDim.x) {
            const int kl = u / n_f;
            const double* r = mv[m] + (size_t)kl * n_f;
            const double v64 = mv[m][u];
            const float v = a.def >= 0 ? __double2float_rn(__ddiv_rn(v64, r[a.def])) : __double2float_rn(v64);
            sv[m][u] = v;
            if (g) g[k0 * n_f + u] = v;
        }
    }
    if (a.mode != kModeSweep) return;
    __syncthreads();
    // each warp takes a contiguous run of (row, target) tasks, so a row's baselines are computed
    // once per warp that touches it instead of once per target
    const int n_t = a.n_t, ntask = nk * n_t, per = (ntask + nw - 1) / nw;
    const int tb = (threadIdx.x >> 5) * per, te = min(ntask, tb + per);
    int row = -1;
    bool base_ok = false;
    RowBase base{};
    for (int task = tb; task < te; ++task) {
        const int kl = task / n_t, t = task - kl * n_t;
        const float* S = sv[0] + (size_t)kl * n_f;
        const float* E = sv[1] + (size_t)kl * n_f;
        if (kl != row) {
            row = kl;
            base_ok = select_baseline(S, E, n_f, a.def, lane, base);
        }
        int c = -1;
        if (base_ok)
            c = select_target(S, E, mv[2] ? sv[2] + (size_t)kl * n_f : nullptr,
                              mv[3] ? sv[3] + (size_t)kl * n_f : nullptr, n_f, a.kind[t], a.frac[t], base,
                              lane);
        if (lane == 0) a.choice[(k0 + kl) * n_t + t] = c;
    }
}

// Standalone selection: one warp per kernel row, rows read from HBM (L1-resident across the
// per-target passes).  Grid-stride over kernels.
__global__ void __launch_bounds__(256) k_select(const __grid_constant__ SelectArgs a) {
    const int lane = threadIdx.x & 31;
    const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
    for (long long k = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); k < a.n_k; k += warps) {
        select_row_warp(a.S + k * a.n_f, a.E + k * a.n_f, nullptr, nullptr, a.n_f, a.def, a.n_t, a.kind, a.frac,
                        a.choice + k * a.n_t, lane);
    }
}

// Pareto front: one warp per kernel, each lane tests its clocks against every clock of the row
// (row read through L1; all lanes read the same j, so the loads are broadcasts).
__global__ void __launch_bounds__(256) k_pareto(const float* __restrict__ S, const float* __restrict__ E,
                                                long long n_k, int n_f, unsigned char* __restrict__ front) {
    const int lane = threadIdx.x & 31;
    const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
    for (long long k = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); k < n_k; k += warps) {
        const float* s = S + k * n_f;
        const float* e = E + k * n_f;
        for (int i0 = 0; i0 < n_f; i0 += 32) {
            const int i = i0 + lane;
            const float si = i < n_f ? __ldg(s + i) : 0.0f, ei = i < n_f ? __ldg(e + i) : 0.0f;
            bool on = i < n_f && valid_pred(si, ei);
            for (int j = 0; j < n_f; ++j) {
                const float sj = __ldg(s + j), ej = __ldg(e + j);
                if (valid_pred(sj, ej) && sj >= si && ej <= ei && (sj > si || ej < ei)) on = false;
            }
            if (i < n_f) front[k * n_f + i] = on ? 1 : 0;
        }
    }
}

__device__ __forceinline__ double target_objective(int kind, float s, float e) {
    const double ds = (double)s, de = (double)e;
    switch (kind) {
        case 0: case 4: case 6: return ds;
        case 1: case 5: case 7: return de;
        case 2: return __ddiv_rn(de, ds);
        default: return __ddiv_rn(__ddiv_rn(de, ds), ds);
    }
}

// Choice error, per kernel (one warp): the truth's choice per target (select_row_warp on the
// ground-truth row, into shared memory), then lane t computes target t's APE and difference.
__global__ void __launch_bounds__(256) k_choice_error(const __grid_constant__ SelectArgs a,
                                                      const int* __restrict__ pred, double* __restrict__ err) {
    __shared__ int truth[8][kMaxTargets];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const long long warps = (long long)gridDim.x * (blockDim.x >> 5);
    for (long long k = (long long)blockIdx.x * (blockDim.x >> 5) + w; k < a.n_k; k += warps) {
        const float* s = a.S + k * a.n_f;
        const float* e = a.E + k * a.n_f;
        select_row_warp(s, e, nullptr, nullptr, a.n_f, a.def, a.n_t, a.kind, a.frac, truth[w], lane);
        __syncwarp();
        if (lane < a.n_t) {
            const int ip = __ldg(pred + k * a.n_t + lane), it = truth[w][lane];
            double ape = CUDART_NAN, diff = CUDART_NAN;
            if (ip >= 0 && ip < a.n_f && it >= 0) {
                const double act = target_objective(a.kind[lane], __ldg(s + it), __ldg(e + it));
                const double pre = target_objective(a.kind[lane], __ldg(s + ip), __ldg(e + ip));
                diff = __dsub_rn(pre, act);
                ape = __ddiv_rn(fabs(diff), fabs(act));
            }
            err[(k * a.n_t + lane) * 2] = ape;
            err[(k * a.n_t + lane) * 2 + 1] = diff;
        }
        __syncwarp();
    }
}

// Per-target reduction (one CTA per target, fixed order): MAPE, RMSE, count.
__global__ void __launch_bounds__(256) k_error_reduce(const double* __restrict__ err, long long n_k, int n_t,
                                                      double* __restrict__ summary) {
    __shared__ double sa[256], ss[256];
    __shared__ long long sc[256];
    const int t = blockIdx.x;
    double a = 0.0, q = 0.0;
    long long c = 0;
    for (long long k = threadIdx.x; k < n_k; k += blockDim.x) {
        const double ape = err[(k * n_t + t) * 2], d = err[(k * n_t + t) * 2 + 1];
        if (!isnan(ape)) { a = __dadd_rn(a, ape); q = __fma_rn(d, d, q); ++c; }
    }
    sa[threadIdx.x] = a; ss[threadIdx.x] = q; sc[threadIdx.x] = c;
    __syncthreads();
    for (int off = blockDim.x / 2; off > 0; off >>= 1) {
        if (threadIdx.x < off) {
            sa[threadIdx.x] += sa[threadIdx.x + off];
            ss[threadIdx.x] += ss[threadIdx.x + off];
            sc[threadIdx.x] += sc[threadIdx.x + off];
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        const double n = (double)sc[0];
        summary[t * 3] = sc[0] ? sa[0] / n : CUDART_NAN;
        summary[t * 3 + 1] = sc[0] ? sqrt(ss[0] / n) : CUDART_NAN;
        summary[t * 3 + 2] = n;
    }
}

// Plan emission: clock index -> MHz (HBM bound: 4 B in, 4 B out per entry).
__global__ void __launch_bounds__(256) k_plan(const int* __restrict__ choice, long long n, const float* __restrict__ freqs,
                                              int n_f, float* __restrict__ mhz) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int c = __ldg(choice + i);
        mhz[i] = (c >= 0 && c < n_f) ? __ldg(freqs + c) : CUDART_NAN_F;
    }
}

}  // namespace syn
