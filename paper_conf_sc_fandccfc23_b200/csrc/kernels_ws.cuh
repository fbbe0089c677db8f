// kernels_ws.cuh — warp-streaming clock-interval sweep (k_sweep_ws), the default fused kernel.
//
// For a fixed kernel only the clock input varies across its n_f evaluations, so every tree is a
// step function of the clock index (P = (k', f)).  The runs of clocks that share a
// leaf are found with restart walks, one root-to-leaf walk per run instead of one per clock:
//
//   walk(lo): follow clock lo's own path (static splits by the kernel's features, clock splits
//             by f_lo <= thr) and keep thr_min = min threshold of the clock splits where the
//             walk went LEFT.  Every clock i >= lo with f_i <= thr_min takes the same path (a
//             clock split that sent f_lo right sends every larger clock right too), and clock
//             #{i : f_i <= thr_min} does not, so the run is [lo, #{i : f_i <= thr_min}).
//             The next walk starts at the run's end.
//
// Walks run on the 2-level block layout (internal.h): one 32-byte block load decides two tree
// levels, so a depth-D walk is ceil(D/2) dependent loads; every lane runs the same number of
// block steps (finished lanes are predicated off), so the 32 lanes of a warp stay in lockstep
// with no stack and no divergent control flow.  Scheduling:
//
//   * one warp owns one (kernel, model) pair for the whole launch; a CTA holds KPC kernels x
//     {speedup, energy} warps; no CTA barrier until the final normalise + select;
//   * each lane walks one tree at a time; when it finishes, it takes the model's next tree in
//     increasing order (ballot + popcount) if that tree's window slot is free;
//   * finished trees park their runs in a ring window of WIN (power of two) slots in shared
//     memory (run-start bitmask over the clock axis, fp32 run values) and the warp applies them
//     strictly in tree order, with p = runs starting in earlier mask words (running popcount):
//         acc[c] += (double) value[ p + popc(mask[c] & lanes<=lane) - 1 ]
//     for the clocks i = 32c + lane this lane owns (fp64 accumulators in registers, _rn adds).
// The accumulation order per evaluation is the oracle's (tree order, fp64), so predictions are
// bit-identical.  Trees with more than vcap runs keep vcap values; their later runs are applied
// through a direct root-to-leaf walk for the clocks involved.
#pragma once
#include "kernels_iv.cuh"

namespace syn {

// 32-bit shared-memory addressing (keeps the hot loops free of generic-address conversions)
__device__ __forceinline__ unsigned su32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ float lds_f(unsigned a) {
    float v;
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ unsigned lds_u(unsigned a) {
    unsigned v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ unsigned lds_u16(unsigned a) {
    unsigned short v;
    asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_f(unsigned a, float v) { asm volatile("st.shared.f32 [%0], %1;" :: "r"(a), "f"(v)); }
__device__ __forceinline__ void sts_u(unsigned a, unsigned v) { asm volatile("st.shared.u32 [%0], %1;" :: "r"(a), "r"(v)); }

// clock_cut on 32-bit shared addresses (see kernels_iv.cuh: exact, the grid is only a hint)
__device__ __forceinline__ int clock_cut_s(unsigned fr_a, unsigned grid_a, float f0, float inv_step,
                                           float thr, int lo, int hi) {
    int b = __float2int_rz((thr - f0) * inv_step);
    b = min(max(b, 0), kGrid);
    int s = min(max((int)lds_u16(grid_a + 2u * b), lo + 1), hi - 1);
    while (s > lo + 1 && !(lds_f(fr_a + 4u * (s - 1)) <= thr)) --s;
    while (s < hi - 1 && lds_f(fr_a + 4u * s) <= thr) ++s;
    return s;
}

__device__ __forceinline__ uint4 ldg_blk(const uint4* p) {
    uint4 r;
    asm volatile("ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// Decide one 2-level block (internal.h layout) already in registers (A = words 0..3, B = 4..7)
// for clock value f: decides at the block's node and at the chosen child, records the smallest
// left-turn clock threshold in tmin, and either moves b to the chosen grandchild block (gslot =
// its slot 0..3) or sets leaf + done.
__device__ __forceinline__ void block_decide(const uint4 A, const uint4 B, int& b, int& gslot, bool& done,
                                             float& leaf, float& tmin, float f, unsigned xrow_a, int F) {
    const unsigned codes = A.w;
    const int cn = (int)(codes & 0xffu);
    const float tn = __uint_as_float(A.x);
    if (cn > F) {                                    // one-leaf tree
        leaf = tn;
        done = true;
        return;
    }
    const float xn = (cn == F) ? f : lds_f(xrow_a + 4u * (unsigned)cn);
    const bool r0 = !(xn <= tn);
    if (cn == F && !r0) tmin = fminf(tmin, tn);
    const float tc = __uint_as_float(r0 ? A.z : A.y);
    const int cc = (int)((codes >> (r0 ? 16 : 8)) & 0xffu);
    if (cc > F) {                                    // the child is a leaf (odd depth)
        leaf = tc;
        done = true;
        return;
    }
    const float xc = (cc == F) ? f : lds_f(xrow_a + 4u * (unsigned)cc);
    const bool r1 = !(xc <= tc);
    if (cc == F && !r1) tmin = fminf(tmin, tc);
    const int slot = (r0 ? 2 : 0) + (r1 ? 1 : 0);
    const unsigned g = r0 ? (r1 ? B.w : B.z) : (r1 ? B.y : B.x);
    if ((codes >> (24 + slot)) & 1u) {              // grandchild is a leaf: value in the slot
        leaf = __uint_as_float(g);
        done = true;
    } else {
        b = (int)g;
        gslot = slot;
    }
}

// Whole 32-byte block in one 256-bit load (sm_100: LDG.E.ENL2.256): one L1 request per block
// instead of two 16-byte ones; blocks are 32-byte aligned.
__device__ __forceinline__ void ldg_blk256(const uint4* p, uint4& A, uint4& B) {
    asm volatile("ld.global.nc.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=r"(A.x), "=r"(A.y), "=r"(A.z), "=r"(A.w), "=r"(B.x), "=r"(B.y), "=r"(B.z), "=r"(B.w)
                 : "l"(p));
}

// One 2-level block step loading the block from global memory (read-only path).
__device__ __forceinline__ void block_step(const uint4* __restrict__ blocks, int& b, bool& done,
                                           float& leaf, float& tmin, float f, unsigned xrow_a, int F) {
    uint4 A, B;
    ldg_blk256(blocks + 2 * (size_t)b, A, B);
    int gs = 0;
    block_decide(A, B, b, gs, done, leaf, tmin, f, xrow_a, F);
}

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned r;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
    return r;
}

// Slot layout (SB bytes): float vals[VS] | uint32 mask[W] | int cnt | int done
template <int CL>
__global__ void __launch_bounds__(256, 4) k_sweep_ws(const __grid_constant__ SweepArgs a) {
    extern __shared__ __align__(16) unsigned char smem[];
    const int KPC = a.tile_k;
    const int n_f = a.n_f, F = a.F, XS = a.xs, W = a.words, VC = a.vcap, VS = a.vs;
    const int WIN = a.win, SB = a.slot_bytes;
    const long long k0 = (long long)blockIdx.x * KPC;
    const int nk = (int)min((long long)KPC, a.n_k - k0);
    float* fr = reinterpret_cast<float*>(smem);
    float* xk = fr + n_f;
    unsigned short* grid = reinterpret_cast<unsigned short*>(xk + KPC * XS);
    unsigned char* slots0 = smem + a.head_bytes;

    const float* gfeat = a.features + k0 * F;
    for (int e = threadIdx.x; e < nk * F; e += blockDim.x) {
        const int r = e / F;
        xk[r * XS + (e - r * F)] = __ldg(gfeat + e);
    }
    for (int r = threadIdx.x; r < nk; r += blockDim.x) {
        xk[r * XS + F] = 0.0f;
        xk[r * XS + F + 1] = CUDART_NAN_F;
    }
    for (int i = threadIdx.x; i < n_f; i += blockDim.x) fr[i] = __ldg(a.freqs + i);
    const float f0 = __ldg(a.freqs);
    const float f_last = __ldg(a.freqs + n_f - 1);
    const float span = f_last - f0;
    const float step = span > 0.0f ? span / (float)kGrid : 1.0f;
    const float inv_step = 1.0f / step;
    for (int b = threadIdx.x; b <= kGrid; b += blockDim.x) {
        const float edge = f0 + (float)b * step;
        int l = 0, h = n_f;
        while (l < h) {
            const int mid = (l + h) >> 1;
            if (__ldg(a.freqs + mid) < edge) l = mid + 1; else h = mid;
        }
        grid[b] = (unsigned short)l;
    }
    for (int j = threadIdx.x; j < (int)(blockDim.x >> 5) * WIN; j += blockDim.x) {   // all slots empty
        int* sl = reinterpret_cast<int*>(slots0 + (size_t)j * SB);
        for (int w = 0; w < W; ++w) sl[VS + w] = 0;
        sl[SB / 4 - 1] = 0;
    }
    __syncthreads();

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int kl = warp >> 1, mdl = warp & 1;
    const DevModel& m = mdl ? a.me : a.ms;
    const int T = (kl < nk && m.forest_weight != 0.0) ? m.n_trees : 0;
    const int BD = m.bdepth;
    const uint4* __restrict__ blocks = m.blocks;
    const float* xrow = xk + kl * XS;
    const unsigned xrow_a = su32(xrow), fr_a = su32(fr), grid_a = su32(grid);
    const unsigned wslots_a = su32(slots0) + (unsigned)(warp * WIN * SB);
    const unsigned mask_off = (unsigned)VS * 4u;
    const unsigned lm_le = (2u << lane) - 1u;
    const unsigned lm_lt = lanemask_lt();
    const int wmask = WIN - 1;

    double acc[CL];
#pragma unroll
    for (int c = 0; c < CL; ++c) acc[c] = 0.0;

    int t = -1;            // tree this lane walks (-1: idle)
    int root = 0, lo = 0, cnt = 0;
    float f_lo = 0.0f, tmin = CUDART_INF_F;
    unsigned slot_a = wslots_a;
    int next = 0, head = 0;
    while (head < T) {
        {   // refill: idle lanes take the next trees in order, inside the window
            const bool want = t < 0;
            const unsigned need = __ballot_sync(0xffffffffu, want);
            const int avail = max(0, min(T, head + WIN) - next);
            const int rank = __popc(need & lm_lt);
            if (want && rank < avail) {
                t = next + rank;
                slot_a = wslots_a + (unsigned)((t & wmask) * SB);   // mask words already zero
                root = __ldg(m.broot + t);
                lo = 0;
                cnt = 0;
                f_lo = lds_f(fr_a);
                tmin = CUDART_INF_F;
            }
            next += min(__popc(need), avail);
        }
        if (__any_sync(0xffffffffu, t >= 0)) {
            // one restart walk from the root block: BD block steps (2 tree levels each)
            float leaf = 0.0f;
            int bk = root;
            bool done = t < 0;
#pragma unroll 2
            for (int d = 0; d < BD; ++d)
                if (!done) block_step(blocks, bk, done, leaf, tmin, f_lo, xrow_a, F);
            if (t >= 0) {
                // run [lo, hi): hi = #{i : f_i <= tmin}  (f_lo <= tmin always)
                const int hi = (tmin < f_last) ? clock_cut_s(fr_a, grid_a, f0, inv_step, tmin, lo, n_f) : n_f;
                if (cnt < VC) sts_f(slot_a + 4u * (unsigned)cnt, leaf);
                const unsigned ma = slot_a + mask_off + 4u * (unsigned)(lo >> 5);
                sts_u(ma, lds_u(ma) | (1u << (lo & 31)));
                ++cnt;
                if (hi >= n_f) {                         // tree done: publish
                    sts_u(slot_a + SB - 8, (unsigned)cnt);
                    __threadfence_block();
                    sts_u(slot_a + SB - 4, 1u);
                    t = -1;
                } else {
                    lo = hi;
                    f_lo = lds_f(fr_a + 4u * (unsigned)hi);
                    tmin = CUDART_INF_F;
                }
            }
        }
        __syncwarp();
        // apply finished trees strictly in tree order
        while (head < T) {
            const unsigned sa = wslots_a + (unsigned)((head & wmask) * SB);
            if (lds_u(sa + SB - 4) == 0u) break;         // same value in every lane
            const int runs = (int)lds_u(sa + SB - 8);
            int p = 0;                                   // runs starting in earlier words
            if (runs <= VC) {
#pragma unroll
                for (int c = 0; c < CL; ++c) {
                    if (c < W) {
                        const unsigned mw = lds_u(sa + mask_off + 4u * c);
                        if (c * 32 + lane < n_f) {
                            const int run = p + __popc(mw & lm_le) - 1;
                            acc[c] = __dadd_rn(acc[c], (double)lds_f(sa + 4u * (unsigned)run));
                        }
                        p += __popc(mw);
                    }
                }
            } else {
                for (int c = 0; c < CL; ++c) {
                    if (c < W) {
                        const unsigned mw = lds_u(sa + mask_off + 4u * c);
                        const int i = c * 32 + lane;
                        if (i < n_f) {
                            const int run = p + __popc(mw & lm_le) - 1;
                            const float v = run < VC ? lds_f(sa + 4u * (unsigned)run)
                                                     : direct_leaf(m, head, xrow, fr[i], F);
                            acc[c] = __dadd_rn(acc[c], (double)v);
                        }
                        p += __popc(mw);
                    }
                }
            }
            __syncwarp();
            if (lane < W) sts_u(sa + mask_off + 4u * lane, 0u);   // slot ready for tree head+WIN
            if (lane == 0) sts_u(sa + SB - 4, 0u);
            __syncwarp();
            ++head;
        }
    }

    __syncthreads();                                     // every warp is done with its slots
    double* mS = reinterpret_cast<double*>(slots0);
    double* mE = mS + (size_t)KPC * n_f;
    float* sS = reinterpret_cast<float*>(mE + (size_t)KPC * n_f);
    float* sE = sS + (size_t)KPC * n_f;
    if (kl < nk) {
        double* out = (mdl ? mE : mS) + (size_t)kl * n_f;
#pragma unroll
        for (int c = 0; c < CL; ++c) {
            const int i = c * 32 + lane;
            if (i < n_f) out[i] = combine(m, acc[c], xrow, fr[i], F);
        }
    }
    __syncthreads();
    finish_tile(a, mS, mE, sS, sE, nk, k0);
}

}  // namespace syn
