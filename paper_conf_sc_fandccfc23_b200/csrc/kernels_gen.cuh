// kernels_gen.cuh — general exact sweep: direct traversal with exact multi-word leaf sums.
//
// The path for every call the tree-major kernels (kernels_tm.cuh) do not take: forests whose
// leaves span more than the int64 fixed-point range (fx_ok = 0), inputs or forests too large for
// k_tm_walk's shared memory (F up to 254, tens of thousands of trees), four-model calls whose
// finish does not fit shared memory, and models without a forest member (linear / SVR only).
// It is the north-star design written plainly: one lane per (kernel, clock) evaluation, lanes of
// a warp along the clock axis (so they share nodes until a clock split), each tree walked from
// its root with predicated gathers of the breadth-first node array.
//
//   k_gen_forest  raw model outputs m(k, f_i) for every model of the call into fp64 scratch:
//                 forest = exact sum of the fp32 leaves rounded once to fp64 (Q8), / T,
//                 plus the linear member (combine()).  Every finite fp32 leaf is v = m * 2^e with
//                 an integer |m| < 2^24 and e >= -s (s from the model's smallest leaf ulp), so
//                 v * 2^s = m * 2^(e+s) is an integer below 2^278.  fx_ok models add it to one
//                 int64; the others add it, split into 32-bit pieces at bit offset e + s, to ten
//                 int64 words (each word receives < 2^32 per tree, so no word overflows for
//                 n_trees < 2^31).  The words are then carry-normalised into a 320-bit two's-
//                 complement integer and rounded once, half to even, to fp64: the correctly
//                 rounded exact sum, whatever the order of the adds — the oracle's math.fsum value.
//   k_gen_finish  SVR members, default-clock normalisation and the per-target argmin
//                 (finish_tile4) for KT kernels per CTA, on the scratch in global memory.
#pragma once
#include "kernels.cuh"

namespace syn {

constexpr int kGenWords = 10;   // 320-bit accumulator: v * 2^s < 2^278, n_trees < 2^31

// Correctly rounded (half to even) fp64 value of the signed integer sum_l w[l] * 2^(32 l), times
// 2^-s.  w[l] are int64 partial sums of 32-bit pieces (any sign); normalised here.
__device__ __forceinline__ double round_words(long long (&w)[kGenWords], int s) {
#pragma unroll
    for (int l = 0; l < kGenWords - 1; ++l) {                  // carry-normalise: w[l] in [0, 2^32)
        const long long c = w[l] >> 32;                        // arithmetic shift (floor)
        w[l] &= 0xffffffffLL;
        w[l + 1] += c;
    }
    const bool neg = w[kGenWords - 1] < 0;                     // |top word| < 2^20: fits 32 bits
    unsigned u[kGenWords];
    unsigned long long carry = 1;
#pragma unroll
    for (int l = 0; l < kGenWords; ++l) {
        const unsigned x = (unsigned)(w[l] & 0xffffffffLL);
        if (neg) {                                             // two's-complement negation
            const unsigned long long y = (unsigned long long)(unsigned)~x + carry;
            u[l] = (unsigned)y;
            carry = y >> 32;
        } else {
            u[l] = x;
        }
    }
    int h = -1;
#pragma unroll
    for (int l = 0; l < kGenWords; ++l)
        if (u[l]) h = l;
    if (h < 0) return 0.0;                                     // exact zero
    const int sh = __clz(u[h]);
    const unsigned long long hi64 = ((unsigned long long)u[h] << 32) | (h >= 1 ? u[h - 1] : 0u);
    const unsigned lo32 = h >= 2 ? u[h - 2] : 0u;
    bool sticky = false;
#pragma unroll
    for (int l = 0; l < kGenWords; ++l)
        if (l < h - 2 && u[l]) sticky = true;
    const unsigned long long win = sh ? ((hi64 << sh) | (unsigned long long)(lo32 >> (32 - sh))) : hi64;
    if (sh ? (unsigned)(lo32 << sh) != 0u : lo32 != 0u) sticky = true;
    int top = 32 * h + 31 - sh;                                // bit index of the leading one
    unsigned long long mant = win >> 11;                       // 53 bits, leading one at bit 52
    const unsigned rb = (unsigned)(win & 0x7ffu);
    if (rb > 0x400u || (rb == 0x400u && (sticky || (mant & 1ull)))) ++mant;
    if (mant == (1ull << 53)) {
        mant >>= 1;
        ++top;
    }
    const int ex = top - 52 - s;                               // |ex| < 1022: 2^ex is a normal fp64
    const double v = __dmul_rn((double)mant, __hiloint2double((ex + 1023) << 20, 0));
    return neg ? -v : v;
}

// Add v * 2^s (v a finite fp32 leaf) to the words (see the header).
__device__ __forceinline__ void add_words(long long (&w)[kGenWords], float v, int s) {
    const unsigned b = __float_as_uint(v);
    const unsigned er = (b >> 23) & 0xffu;
    const unsigned long long m = er ? ((b & 0x7fffffu) | 0x800000u) : (b & 0x7fffffu);
    if (!m) return;
    const int p = (er ? (int)er - 150 : -149) + s;             // >= 0 by the choice of s
    const unsigned long long x = m << (p & 31);                // < 2^55
    const long long lo = (long long)(x & 0xffffffffull), hi = (long long)(x >> 32);
    const int l = p >> 5;
    if (b >> 31) {
        w[l] -= lo;
        w[l + 1] -= hi;
    } else {
        w[l] += lo;
        w[l + 1] += hi;
    }
}

struct GenArgs {
    SweepArgs s;
    double* mv;       // [NM][nks][n_f] raw model outputs of the slab (fp64)
    float* sv;        // [NM][nks][n_f] fp32 scratch of finish_tile4
    long long slab0;  // global index of the slab's first kernel
    int nks;          // kernels in the slab
    int nm;           // models in the call (2 or 4)
};

__global__ void __launch_bounds__(256) k_gen_forest(const __grid_constant__ GenArgs g) {
    const SweepArgs& a = g.s;
    const int n_f = a.n_f, F = a.F;
    const long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (u >= (long long)g.nks * n_f) return;
    const int kl = (int)(u / n_f), i = (int)(u - (long long)kl * n_f);
    const float* xrow = a.features + (g.slab0 + kl) * F;
    const float f = __ldg(a.freqs + i);
    for (int mi = 0; mi < g.nm; ++mi) {
        if (!model_present(a, mi)) continue;
        const DevModel& m = model_of(a, mi);
        double forest_sum = 0.0;
        if (m.forest_weight != 0.0) {
            long long acc = 0;
            long long w[kGenWords];
#pragma unroll
            for (int l = 0; l < kGenWords; ++l) w[l] = 0;
            const bool fx = m.fx_ok != 0;
            for (int t = 0; t < m.n_trees; ++t) {
                int idx = __ldg(&m.trees[t].x);
                uint2 nd = ldg_node(m.nodes + idx);
                int code = (int)(nd.y & 0xffu);
                while (code <= F) {                            // x <= thr goes left (Q9)
                    const float x = code == F ? f : __ldg(xrow + code);
                    idx += ((int)nd.y >> kCodeBits) + (x <= __uint_as_float(nd.x) ? 0 : 1);
                    nd = ldg_node(m.nodes + idx);
                    code = (int)(nd.y & 0xffu);
                }
                const float v = __uint_as_float(nd.x);
                if (fx) acc += __double2ll_rn(__dmul_rn((double)v, m.fx_scale));   // exact
                else add_words(w, v, m.fx_s);
            }
            forest_sum = fx ? __dmul_rn(__ll2double_rn(acc), m.fx_inv) : round_words(w, m.fx_s);
        }
        g.mv[((size_t)mi * g.nks + kl) * n_f + i] = combine(m, forest_sum, xrow, f, F);
    }
}

__global__ void __launch_bounds__(256) k_gen_finish(const __grid_constant__ GenArgs g) {
    const SweepArgs& a = g.s;
    const int KT = a.tile_k, n_f = a.n_f;
    const int k0s = blockIdx.x * KT;
    const int nk = min(KT, g.nks - k0s);
    double* mv[4];
    float* sv[4];
    for (int m = 0; m < 4; ++m) {
        const bool present = m < g.nm && model_present(a, m);
        mv[m] = present ? g.mv + ((size_t)m * g.nks + k0s) * n_f : nullptr;
        sv[m] = present ? g.sv + ((size_t)m * g.nks + k0s) * n_f : nullptr;
    }
    finish_tile4(a, mv, sv, nk, g.slab0 + k0s);
}

}  // namespace syn
