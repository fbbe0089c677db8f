// kernels_tr.cuh — tree-resident resume-walk sweep (k_tr_walk), the walk half of the default
// fused path when every tree of the call fits a shared-memory tree buffer.
//
// It computes exactly what k_tm_walk computes (kernels_tm.cuh): per (kernel, model) the exact
// fixed-point difference array over the clock axis of the leaves each clock reaches (DESIGN.md
// Q8), by resume walks over the clock-cut 2-level blocks, with one 64-bit global
// reduction per run.  k_tm_finish then scans, rounds, combines and selects as for k_tm_walk.
// What changes is where the tree lives while it is walked (round-1 ncu of k_tm_walk: the L1 data
// pipe at 83% of peak, ~5e8 of its 8e8 wavefronts per c3 slab being scattered 32-B global block
// loads, one per lane and step) and how work reaches the lanes:
//
//  * Units.  A unit is (one tree, one chunk of P kernels); units are numbered chunk-major
//    (u = chunk * TT + tree) and every CTA (one per SM) owns a contiguous unit range.
//  * Staging by bulk copy (cp.async.bulk + mbarrier complete_tx: the TMA engine, no register
//    round trip).  Trees: a kTrNB-deep ring, unit j in buffer j % kTrNB, from the tree-resident
//    layout (k_tr_layout, once per (model, clock table)): per tree the 16-B heads
//    {thr(n), thr(c0), thr(c1), codes} of its blocks, then their 16-B grandchild quads, references
//    tree-local; a step loads one head and the ONE grandchild word it takes.  Features: the
//    chunk's [F][P] block of a transposed copy (k_tr_feat), one buffer per CTA.
//  * Task pools.  A task is one kernel of the unit.  Lane l takes the kernels l, l + 32, ... of
//    the chunk from a pool shared by the NT / 32 lanes with lane index l (a shared counter per
//    (buffer, lane index)): feature reads x[code][kernel] hit bank l, conflict-free, and lanes
//    that drew short walks simply draw more.
//  * Per-lane progression.  A lane whose pool is empty counts itself out of the unit's buffer and
//    moves on to unit j + 1 at once (waiting only if that tree has not landed, mbarrier
//    test_wait).  The lane that counts the buffer's last walker out stages unit j + kTrNB into it.
//    At a chunk boundary the last lane out of the chunk stages the next chunk's features.  No CTA
//    barrier anywhere after the prologue.
//  * The step, the record stack (kTmS shallowest records), clock cuts, folded leaves, int32
//    fixed-point leaves and the REDG difference-array adds are k_tm_walk's (kernels_tm.cuh; models
//    whose leaves need int64 fixed point take k_tm_walk).
#pragma once
#include "kernels_tm.cuh"
#include "kernels_svr.cuh"

namespace syn {

constexpr int kTrNB = 2;         // tree buffers per CTA
constexpr int kTrNT = 1024;      // k_tr_walk threads per CTA (one CTA per SM)

struct TrArgs {
    TmArgs tm;                   // D, slab, models; k_tm_finish runs on tm afterwards
    const uint4* trb[4];         // per model: tree-resident clock-cut layout (null without forest)
    const float* featT;          // [nchunks][F][P] transposed features of the slab (k_tr_feat)
    int tree_smem;               // bytes of one tree buffer (>= 32 x blocks of any tree, 128-aligned)
    int P;                       // kernels per chunk (multiple of 32)
    int nchunks;                 // ceil(nks / P)
};

// Tree-resident copy of clock-cut blocks: tree t's blocks [s, e) become heads [2s, 2s + nb) and
// grandchild quads [2s + nb, 2s + 2nb) (uint4 units), grandchild block references minus s.
__global__ void __launch_bounds__(256) k_tr_layout(const uint4* __restrict__ cut, const int* __restrict__ broot,
                                                   int n_trees, long long nblk, uint4* __restrict__ out) {
    const int t = blockIdx.x;
    const long long s = broot[t], e = t + 1 < n_trees ? broot[t + 1] : nblk;
    const long long nb = e - s;
    for (long long i = threadIdx.x; i < nb; i += blockDim.x) {
        const uint4 A = cut[2 * (s + i)];
        uint4 B = cut[2 * (s + i) + 1];
        const unsigned lm = A.w >> 24;
        const unsigned su = (unsigned)s;
        if (!(lm & 1u)) B.x -= su;
        if (!(lm & 2u)) B.y -= su;
        if (!(lm & 4u)) B.z -= su;
        if (!(lm & 8u)) B.w -= su;
        out[2 * s + i] = A;
        out[2 * s + nb + i] = B;
    }
}

// Transposed features of a slab: featT[chunk][c][col] = features[slab0 + chunk * P + col][c]
// (zero past the slab end).
__global__ void __launch_bounds__(256) k_tr_feat(const float* __restrict__ features, long long slab0, int nks,
                                                 int F, int P, int nchunks, float* __restrict__ featT) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;   // (chunk, c, col)
    const long long n = (long long)nchunks * F * P;
    if (i >= n) return;
    const int col = (int)(i % P);
    const long long r = i / P;
    const int c = (int)(r % F);
    const long long k = (r / F) * P + col;
    featT[i] = k < nks ? __ldg(features + (slab0 + k) * F + c) : 0.0f;
}

__device__ __forceinline__ bool mbar_test(unsigned long long* bar, unsigned parity) {
    unsigned ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}" : "=r"(ok) : "r"((unsigned)__cvta_generic_to_shared(bar)), "r"(parity) : "memory");
    return ok != 0;
}

template <int NT>
__global__ void __launch_bounds__(NT, 1) k_tr_walk(const __grid_constant__ TrArgs r) {
    const TmArgs& t = r.tm;
    const SweepArgs& a = t.s;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) unsigned long long full[kTrNB], fbar;
    __shared__ int done[kTrNB], fdone;
    __shared__ int cnt[kTrNB][32];
    __shared__ int2 meta[kTrNB];                                              // {blocks, D slot offset}
    const int n_f = a.n_f, F = a.F, P = r.P;
    float* xs = reinterpret_cast<float*>(smem + kTrNB * r.tree_smem);       // [F][P] chunk features
    int* stk_b = reinterpret_cast<int*>(xs + (size_t)F * P);                // [kTmS][NT] record blocks
    float* stk_c = reinterpret_cast<float*>(stk_b + kTmS * NT);             // [kTmS][NT] record cuts
    int* const sb = stk_b + threadIdx.x;
    float* const sc = stk_c + threadIdx.x;
    const int lane = threadIdx.x & 31;
    const int Fm1 = max(F - 1, 0);

    const int T0 = da_trees(a, 0), T1 = da_trees(a, 1), T2 = t.nm > 2 ? da_trees(a, 2) : 0,
              T3 = t.nm > 2 ? da_trees(a, 3) : 0;
    const int c1 = T0, c2 = c1 + T1, c3 = c2 + T2, TT = c3 + T3;
    const long long U = (long long)r.nchunks * TT;
    const long long u0 = (long long)blockIdx.x * U / gridDim.x, u1 = (long long)(blockIdx.x + 1) * U / gridDim.x;
    const int J = (int)(u1 - u0);
    const unsigned fbytes = 4u * (unsigned)F * (unsigned)P;

    // stage unit jj of this CTA's range into buffer jj % kTrNB (one thread)
    auto stage = [&](int jj) {
        const long long v = u0 + jj;
        const int tti = (int)(v % TT);
        const int mi = tti < c1 ? 0 : tti < c2 ? 1 : tti < c3 ? 2 : 3;
        const int lt = tti - (mi == 0 ? 0 : mi == 1 ? c1 : mi == 2 ? c2 : c3);
        const DevModel& m = da_model(a, mi);
        const int s = __ldg(m.broot + lt);
        const int e = lt + 1 < m.n_trees ? __ldg(m.broot + lt + 1) : m.nblk;
        const int b = jj % kTrNB;
        meta[b] = make_int2(e - s, t.slot_of[mi] * n_f);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&full[b], 32u * (unsigned)(e - s));
        bulk_g2s(smem + (size_t)b * r.tree_smem, r.trb[mi] + 2 * (size_t)s, 32u * (unsigned)(e - s), &full[b]);
    };
    auto stage_feat = [&](long long ch) {                                   // one thread
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&fbar, fbytes);
        bulk_g2s(xs, r.featT + (size_t)ch * F * P, fbytes, &fbar);
    };
    if (threadIdx.x == 0) {
        for (int b = 0; b < kTrNB; ++b) {
            mbar_init(&full[b], 1);
            done[b] = 0;
        }
        mbar_init(&fbar, 1);
        fdone = 0;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        if (J > 0 && F > 0) stage_feat(u0 / TT);
        for (int jj = 0; jj < min(kTrNB, J); ++jj) stage(jj);
    }
    for (int q = threadIdx.x; q < kTrNB * 32; q += NT) cnt[q >> 5][q & 31] = 0;
    __syncthreads();
    if (J <= 0) return;

    // lane state: unit j (chunk ch, its features' load parity fpar), task (kernel col of the chunk)
    // (flags, not a state variable: a switch compiles to an indexed jump table, a divergent
    // constant-bank load per iteration)
    bool need_unit = true, need_task = false, walking = false, fin = false;
    int j = 0;
    long long ch = u0 / TT;
    unsigned fpar = 0;
    const uint4* heads = nullptr;                                            // current tree (shared)
    const unsigned* quads = nullptr;
    int slotoff = 0;
    const float* xk = xs;                                                    // column of the task's kernel
    long long* drow = t.D;
    int bk = 0, lo = 0, sn = 0;
    float f_lo = 0.5f, tmin = CUDART_INF_F;
    int vprev = 0;

    while (__any_sync(0xffffffffu, !fin)) {
        if (need_unit) {
            const int b = j % kTrNB;
            if (mbar_test(&full[b], (unsigned)((j / kTrNB) & 1)) && (F == 0 || mbar_test(&fbar, fpar))) {
                const int2 mt = meta[b];
                heads = reinterpret_cast<const uint4*>(smem + (size_t)b * r.tree_smem);
                quads = reinterpret_cast<const unsigned*>(heads + mt.x);
                slotoff = mt.y;
                need_unit = false;
                need_task = true;
            }
        }
        if (need_task) {
            const int b = j % kTrNB;
            const int col = lane + 32 * atomicAdd(&cnt[b][lane], 1);
            const long long k = ch * P + col;                                 // slab-relative kernel
            if (col < P && k < t.nks) {
                xk = xs + col;
                drow = t.D + (size_t)k * t.nslot * n_f + slotoff;
                bk = 0;
                lo = 0;
                sn = 0;
                f_lo = 0.5f;
                tmin = CUDART_INF_F;
                vprev = 0;
                need_task = false;
                walking = true;
            } else {
                // pool empty: count out of the buffer (the last one out stages unit j + kTrNB)
                __threadfence_block();
                if (atomicAdd(&done[b], 1) == NT - 1) {
                    for (int q = 0; q < 32; ++q) cnt[b][q] = 0;
                    done[b] = 0;
                    if (j + kTrNB < J) stage(j + kTrNB);
                }
                ++j;
                const bool last = j == J;
                if (last || (u0 + j) % TT == 0) {
                    // leaving chunk ch: the last one out stages the next chunk's features
                    if (atomicAdd(&fdone, 1) == NT - 1) {
                        fdone = 0;
                        if (!last && F > 0) stage_feat(ch + 1);
                    }
                    ++ch;
                    fpar ^= 1u;
                }
                need_task = false;
                fin = last;
                need_unit = !last;
            }
        }
        if (walking) {
            // one 2-level block step (tm_step on the clock-cut words): head, the three candidate
            // inputs (the clock from a register), then the one grandchild word taken
            const int cur = bk;
            const uint4 A = heads[cur];
            const unsigned codes = A.w;
            const int cn = (int)(codes & 0xffu), k0c = (int)((codes >> 8) & 0xffu), k1c = (int)((codes >> 16) & 0xffu);
            const float xn_s = xk[(size_t)min(cn, Fm1) * P];
            const float x0_s = xk[(size_t)min(k0c, Fm1) * P];
            const float x1_s = xk[(size_t)min(k1c, Fm1) * P];
            const bool clk_n = codes & kClkN;
            const bool l0 = (clk_n ? f_lo : xn_s) <= __uint_as_float(A.x);
            const unsigned tcb = l0 ? A.y : A.z;
            const bool clk_c = codes & (l0 ? kClkC0 : kClkC1);
            const bool l1 = (clk_c ? f_lo : (l0 ? x0_s : x1_s)) <= __uint_as_float(tcb);
            const float cbn = (l0 && clk_n) ? __uint_as_float(A.x) : CUDART_INF_F;
            const float cbc = (l1 && clk_c) ? __uint_as_float(tcb) : CUDART_INF_F;
            const float cb = fminf(cbn, cbc);
            const int slot = (l0 ? 0 : 2) + (l1 ? 0 : 1);
            const unsigned g = quads[4 * cur + slot];
            const bool at_leaf = (codes >> (24 + slot)) & 1u;
            bk = (int)g;
            if (cb < tmin) {                                                 // new record
                if (sn < kTmS) {
                    sb[sn * NT] = cur;
                    sc[sn * NT] = cb;
                    ++sn;
                }
                tmin = cb;
            }
            if (at_leaf) {
                // run [lo, hi): D[lo] += v - v_prev (exact int64 of int32 fixed-point leaves)
                const int hi = tmin < CUDART_INF_F ? (int)tmin : n_f;
                atomicAdd(reinterpret_cast<unsigned long long*>(drow + lo),
                          (unsigned long long)((long long)(int)g - (long long)vprev));
                vprev = (int)g;
                if (hi < n_f) {
                    --sn;
                    bk = sb[sn * NT];
                    tmin = sn > 0 ? sc[(sn - 1) * NT] : CUDART_INF_F;
                    lo = hi;
                    f_lo = (float)hi + 0.5f;
                } else {
                    walking = false;
                    need_task = true;
                }
            }
        }
    }
}

}  // namespace syn
