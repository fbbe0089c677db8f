// kernels_tm.cuh — tree-major resume-walk sweep (k_tm_walk + k_tm_finish), the default fused path.
//
// Computes, per (kernel, model), the exact fixed-point sum over trees of the leaf each clock
// reaches (Q8), accumulated as a difference array over the clock axis, then the forest
// mean, linear / SVR members, default-clock normalisation and the per-target masked argmin (PAPER
// L253-L271, L316-L322).  Needs every forest within the int64 fixed-point range (fx_ok) and the
// shared-memory limits checked by the host (tm_eligible); kernels_gen.cuh takes the rest.  The
// work is laid on the machine to cut L1 wavefronts, the resource a kernel-major walk saturates:
//
//  * Tree-major lanes.  A lane task is one (kernel, model, tree) (or a clock sub-range of one,
//    SUB).  Tasks are numbered
//      j = ((kernel block) * TT + tree) * KB + kernel-in-block
//    and every CTA owns a contiguous range of j, so the lanes of an SM walk the SAME few trees for
//    up to KB different kernels at once: the SM's L1 holds those trees (block loads hit L1 ~97 %
//    of the time on c3), the 32 lanes of a warp load blocks of one tree, and lines are reused by
//    every kernel of the block.  Within a CTA, lane l of every warp takes the tasks j = l mod 32
//    in order from its pool's shared counter (per-lane-index task pools), so short walks are
//    balanced by taking the remaining tasks and a warp's kernels stay distinct mod 32.
//
//  * Resume walks.  For a fixed kernel a tree is a step function of the clock index.  walk(lo)
//    follows clock lo's path; the run is [lo, hi) with hi = #{i : f_i <= thr} minimised over the
//    clock splits where the walk went LEFT.  The next clock hi follows the same path down to the
//    first split that sends it right: the shallowest left-turn split whose cut equals hi (static
//    splits do not depend on the clock, right turns stay right for a larger clock, and a left
//    turn with a larger cut stays left).  So each lane keeps the prefix-minimum ("record") cuts
//    of its path with their blocks, one entry per block, deepest on top: the next walk resumes at
//    the top record's block (popped; the block is re-decided), and the new bound is the next
//    record.  The stack keeps the kTmS shallowest records (a depth-12 path has at most 6 blocks);
//    deeper ones are not pushed, which stays exact: resuming at any ancestor block of the path
//    re-walks the same path down to the split where clock hi turns right.  On the bench forests
//    this fetches 0.47x the blocks of root restarts.
//
//  * Clock cuts instead of clock values.  For a given clock table every clock-split threshold
//    thr is replaced (k_cut_blocks, once per (model, clock table)) by its cut index
//    c = #{i : f_i <= thr}, an integer exact in fp32, and clock i enters the walk as the value
//    i + 0.5: f_i <= thr  <=>  i < c  <=>  i + 0.5 <= c, so every decision is unchanged.  The
//    run end is then simply hi = min c over the left-turn clock splits (no search in the clock
//    table), and split e is where clock hi turns right iff c_e < hi + 0.5.
//
//  * Step-level lockstep.  Every loop iteration is one 2-level block step for every busy lane; a
//    lane that reaches a leaf closes its run and resumes in the same iteration, so walks of
//    different lengths do not idle lanes.  The kernel block's static features sit once per
//    segment in a transposed shared table [F + 2][KB] (kernel kk in bank kk mod 32 of every row),
//    the walked clock is a register, and clock splits and leaves are flagged in the block
//    (k_cut_blocks); a step reads the node's input, decides, then reads the taken child's.
//
//  * Accumulation in L2.  Run j of a (kernel, model, tree) adds v_j - v_{j-1} to
//    D[kernel][slot][lo_j] with one 64-bit global reduction (exact, order-free; run 0 adds v_0).
//    No shared-memory difference arrays (a slab's D rows are tens of MB).  k_tm_finish then scans
//    each D row (exact int64 prefix sum = the exact leaf sum per clock), rounds it once, combines
//    the members and runs finish_tile4; it zeroes D as it reads it, so the next call starts from
//    zeros without a memset.
#pragma once
#include "kernels.cuh"

namespace syn {

constexpr int kTmS = 6;          // record-stack entries per lane (a depth-12 path has <= 6 blocks)

// Clock-cut block words (k_cut_blocks output; the layout of internal.h with two additions):
//   word 3 bits 28/29/30: node / child 0 / child 1 splits on the clock (code == F)
//   leaves folded into grandchild slots: a child that is a leaf (code F + 1) has both its
//   grandchild slots set to its value with their leafmask bits, and a one-leaf tree has all four
//   (children then read feature row F + 1 of any value: both outcomes reach the same leaf).
// So a step reaches a leaf exactly when the leafmask bit of the slot it takes is set, and the
// leaf value is that slot's word.
constexpr unsigned kClkN = 1u << 28, kClkC0 = 1u << 29, kClkC1 = 1u << 30;

struct TmArgs {
    SweepArgs s;                 // models, clocks, targets, outputs of the whole call
    long long* D;                // [nks][nslot][n_f] int64 difference arrays, zero on entry
    long long slab0;             // global index of the slab's first kernel
    long long n_tasks;           // ceil(nks / kb) * TT * kb lane tasks
    int nks;                     // kernels in this slab
    int kb;                      // kernels per feature block (power of two, 32..256)
    int kb_log2;
    int nslot;                   // D slots = models with a forest member
    int slot_of[4];              // model -> D slot, -1 without forest
    int nm;                      // models in the call (2 or 4)
    int nsub;                    // smode 1: clock sub-ranges per (kernel, tree) (tiny batches)
    int smode;                   // units: 0 one per tree, 1 nsub per tree, 2 per-tree split (tsplit)
    int units;                   // units per kernel block (tasks per kernel)
    int dyn;                     // k_tm_walk: tasks from a shared counter
    int lpt;                     // the models' roots are in expected-cost order (broot_lpt): tree
                                 // ranges are not contiguous in the blocks, so the prefetch differs
};

// One 2-level block step on clock-cut words (A = {thr(n), thr(c0), thr(c1), codes}, grandchild
// words B): a node's input is the kernel's static feature (shared-memory column at xb of the
// block's feature table [F + 2][KB], row stride rs = 4 KB bytes; row F + 1 = 0 serves folded
// leaves) or, for clock splits (flag bits), the walked clock clk.  The node is decided first and
// only the taken child's input is read.  Returns
// the grandchild word taken; *cb = smallest cut of the block's left-turn clock splits (+inf if
// none), *leaf = the word is a leaf value.
__device__ __forceinline__ unsigned tm_step(const uint4& A, const uint4& B, unsigned xb, unsigned rs, float clk,
                                            float& cb, bool& leaf) {
    const unsigned codes = A.w;
    // the node's input, its decision, then only the taken child's input (two shared-memory reads
    // per step instead of three: measured c3 walk -2 %, c2 / c5 -3 %)
    const float fn = lds_f(xb + rs * (codes & 0xffu));
    const float xn = (codes & kClkN) ? clk : fn;
    const bool l0 = xn <= __uint_as_float(A.x);
    const float fc = lds_f(xb + rs * ((codes >> (l0 ? 8 : 16)) & 0xffu));
    const unsigned cfl = l0 ? kClkC0 : kClkC1;
    const float xc = (codes & cfl) ? clk : fc;
    const unsigned tcb = l0 ? A.y : A.z;
    const bool l1 = xc <= __uint_as_float(tcb);
    const float cbn = (l0 && (codes & kClkN)) ? __uint_as_float(A.x) : CUDART_INF_F;
    const float cbc = (l1 && (codes & cfl)) ? __uint_as_float(tcb) : CUDART_INF_F;
    cb = fminf(cbn, cbc);
    const int slot = (l0 ? 0 : 2) + (l1 ? 0 : 1);
    leaf = (codes >> (24 + slot)) & 1u;
    return l0 ? (l1 ? B.x : B.y) : (l1 ? B.z : B.w);
}

__device__ __forceinline__ int d0_units(const SweepArgs& a) { return model_of(a, 0).units_split; }

// Per-tree task record in shared memory: everything a task start needs in one 16-byte load.
struct __align__(16) TmTree {
    int root;            // root block
    int slot_off;        // D slot offset of the tree's model (slot * n_f)
    const uint4* blocks; // the model's clock-cut blocks
};

// FXALL: every forest of the call has int32 fixed-point leaves (no int64 conversion path).
// SUB: a task is (kernel, unit) with a unit = (tree, clock sub-range [lo, end)) from a unit table
// in shared memory (t.smode 1: every tree in t.nsub equal sub-ranges, tiny batches; 2: each tree
// in its tsplit sub-ranges, small batches); otherwise a unit is a whole tree.
// LPT: the models' roots are the expected-cost order (broot_lpt, t.lpt): a compile-time variant so
// that the other launches keep their code unchanged.
template <int NT, bool FXALL, bool SUB, bool LPT = false>
__global__ void __launch_bounds__(NT, 1024 / NT) k_tm_walk(const __grid_constant__ TmArgs t) {
    const SweepArgs& a = t.s;
    extern __shared__ __align__(16) unsigned char smem[];
    asm volatile("griddepcontrol.launch_dependents;");                       // k_tm_finish may launch early
    const int n_f = a.n_f, F = a.F, KB = t.kb, KBL = t.kb_log2;
    TmTree* stree = reinterpret_cast<TmTree*>(smem);                         // [TT] task records
    const int T0 = trees_of(a, 0), T1 = trees_of(a, 1), T2 = t.nm > 2 ? trees_of(a, 2) : 0,
              T3 = t.nm > 2 ? trees_of(a, 3) : 0;
    const int c1 = T0, c2 = c1 + T1, c3 = c2 + T2, TT = c3 + T3;
    int* stk_b = reinterpret_cast<int*>(stree + TT);                         // [kTmS][NT] record blocks
    float* stk_c = reinterpret_cast<float*>(stk_b + kTmS * NT);              // [kTmS][NT] record cuts
    float* xs = stk_c + kTmS * NT;                                           // [F + 2][KB] block's features
    int2* units = reinterpret_cast<int2*>(xs + (size_t)(F + 2) * KB);         // [U] (SUB) {tree, lo | end << 16}
    unsigned char* smodel = reinterpret_cast<unsigned char*>(units + (SUB ? t.units : 0));   // [TT] (!FXALL)
    __shared__ int s_pool[32];                                               // dynamic mode: next task per pool
    __shared__ int s_nblk[4];                                                // per model: blocks in all,
    __shared__ int s_fx[4];                                                  // int32 leaves,
    __shared__ double s_scale[4];                                            // fixed-point scale
    const unsigned sb_a = su32(stk_b) + 4u * threadIdx.x, sc_a = su32(stk_c) + 4u * threadIdx.x;
    constexpr unsigned kEnt = 4u * NT;                                       // bytes between stack entries
    const unsigned xs_a = su32(xs);
    unsigned rs;                                                             // feature row stride (bytes),
    asm volatile("mov.u32 %0, %1;" : "=r"(rs) : "r"(4u * (unsigned)KB));     // kept in a register

    const int U = SUB ? t.units : TT;
    const long long per_kb = (long long)U * KB;
    for (int q = threadIdx.x; q < TT; q += NT) {
        const int mi = q < c1 ? 0 : q < c2 ? 1 : q < c3 ? 2 : 3;
        const DevModel& d = model_of(a, mi);
        TmTree r;
        r.root = __ldg(d.broot + (q - (mi == 0 ? 0 : mi == 1 ? c1 : mi == 2 ? c2 : c3)));
        r.slot_off = t.slot_of[mi] * n_f;
        r.blocks = d.blocks;
        stree[q] = r;
        if (!FXALL) smodel[q] = (unsigned char)mi;
        if (SUB) {
            int u0, ns;
            if (t.smode == 1) {
                u0 = q * t.nsub;
                ns = t.nsub;
            } else {
                const int mbase = (mi >= 1 ? d0_units(a) : 0) + (mi >= 2 ? model_of(a, 1).units_split : 0) +
                                  (mi >= 3 ? model_of(a, 2).units_split : 0);
                const int2 sp = __ldg(d.tsplit + (q - (mi == 0 ? 0 : mi == 1 ? c1 : mi == 2 ? c2 : c3)));
                u0 = mbase + sp.x;
                ns = sp.y;
            }
            for (int sub = 0; sub < ns; ++sub)
                units[u0 + sub] = make_int2(q, (sub * n_f / ns) | (((sub + 1) * n_f / ns) << 16));
        }
    }
    if (threadIdx.x < 4) {
        const int m = threadIdx.x;
        if (m < 2 || t.nm > 2) {
            const DevModel& d = model_of(a, m);
            s_nblk[m] = d.nblk;
            s_fx[m] = d.fx32;
            s_scale[m] = d.fx_scale;
        }
    }
    const long long r0 = (long long)blockIdx.x * t.n_tasks / gridDim.x;
    const long long r1 = (long long)(blockIdx.x + 1) * t.n_tasks / gridDim.x;
    const int lane = threadIdx.x & 31;
    const size_t row = (size_t)t.nslot * n_f;                                // D entries per kernel

    for (long long s0 = r0; s0 < r1;) {
        const long long kbi = s0 / per_kb;
        const long long s1 = min(r1, (kbi + 1) * per_kb);
        const int kbase = (int)(kbi * KB);                                   // slab-relative
        const int nvalid = min(KB, t.nks - kbase);
        // the kernel block's static features into shared memory, once per segment, transposed
        // ([feature][kernel]: lanes on kernels distinct mod 32 read distinct banks); row F + 1 = 0
        // for folded leaves (row F, the clock, is never read: clock splits take clk)
        __syncthreads();                                                     // previous segment done
        const float* gblk = a.features + (t.slab0 + kbase) * F;
        for (int e = threadIdx.x; e < nvalid * F; e += NT) {
            const int r = e / F;
            xs[(e - r * F) * KB + r] = __ldg(gblk + e);
        }
        for (int r = threadIdx.x; r < KB; r += NT) xs[(F + 1) * KB + r] = 0.0f;
        const int seg0 = (int)(s0 - kbi * per_kb), seg1 = (int)(s1 - kbi * per_kb);
        // pull the blocks of the segment's first trees (at most 8) into L2 with bulk prefetches
        // (one per model's contiguous tree range), so the first walks of a cold model do not
        // serialise DRAM misses; later trees of a long range arrive while the first are walked
        if (LPT && threadIdx.x == 0) {
            // cost-ordered roots: CTA c pulls its share of every model's blocks instead (together
            // the CTAs prefetch each model once)
            for (int mi = 0; mi < 4; ++mi) {
                if (!(mi == 0 ? T0 : mi == 1 ? T1 : mi == 2 ? T2 : T3)) continue;
                const long long nb = s_nblk[mi];
                const long long b0 = nb * blockIdx.x / gridDim.x, b1 = nb * (blockIdx.x + 1) / gridDim.x;
                const char* p = reinterpret_cast<const char*>(model_of(a, mi).blocks + 2 * (size_t)b0);
                size_t left = (size_t)(b1 - b0) * 32;
                while (left > 0) {
                    const unsigned n = (unsigned)min(left, (size_t)1 << 20);
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(p), "r"(n) : "memory");
                    p += n;
                    left -= n;
                }
            }
        } else if (!LPT && threadIdx.x == 0) {
            const int ta = SUB ? units[seg0 >> KBL].x : seg0 >> KBL;
            const int tb = min(ta + 7, SUB ? units[(seg1 - 1) >> KBL].x : (seg1 - 1) >> KBL);
            int u = ta;
            while (u <= tb) {
                const int mi = u < c1 ? 0 : u < c2 ? 1 : u < c3 ? 2 : 3;
                const int mend = mi == 0 ? c1 : mi == 1 ? c2 : mi == 2 ? c3 : TT;   // model's trees end
                const int v = min(tb + 1, mend);
                const int b0 = stree[u].root;
                const int b1 = v < mend ? stree[v].root : s_nblk[mi];
                if (b1 > b0) {
                    const char* p = reinterpret_cast<const char*>(stree[u].blocks + 2 * (size_t)b0);
                    size_t left = (size_t)(b1 - b0) * 32;
                    while (left > 0) {
                        const unsigned n = (unsigned)min(left, (size_t)1 << 20);
                        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(p), "r"(n) : "memory");
                        p += n;
                        left -= n;
                    }
                }
                u = v;
            }
        }
        // first task of each pool (tasks j = l mod 32) at or after seg0
        const int base_l = seg0 + (((lane - seg0) % 32) + 32) % 32;
        if (threadIdx.x < 32) s_pool[lane] = base_l + NT;
        __syncthreads();
        // Static lane streams (t.dyn == 0): task j (tree j / KB, kernel-in-block j % KB) of the
        // segment goes to lane j % 32 of warp (j / 32) % NW, so every task of a lane has the same
        // kernel and its trees advance by NT / KB.  Dynamic (t.dyn): per-lane-index pools, lane l
        // of every warp takes the tasks j = l mod 32 in task order from its pool's counter (one
        // conflict-free shared atomic per task), so the CTA's lanes stay within a few trees (L1-
        // resident), lanes that drew short walks take the remaining tasks, and the kernels of a
        // warp's lanes stay distinct mod 32 (conflict-free feature reads: kernel kk sits in bank
        // kk mod 32 of every feature row).  Either way a task start only sets registers: the
        // kernel's features are already in shared memory.
        int q;
        if (t.dyn) {
            q = base_l + 32 * (threadIdx.x >> 5);
        } else {
            const int nw = NT / 32, w = threadIdx.x >> 5;
            const int g0 = seg0 >> 5;
            const int g = g0 + ((w - g0 % nw) + nw) % nw;
            q = 32 * g + lane;
            if (q < seg0) q += NT;
        }
        long long* const dk = t.D + (size_t)kbase * row;                     // the block's D rows
        long long* drow = dk;
        const uint4* blocks = nullptr;
        double scale = 1.0;
        bool fxm = true;                                                     // this model's leaves are int32
        int bk = 0, lo = 0, sn = 0, end = n_f;
        unsigned xb = xs_a;
        float tmin = CUDART_INF_F, clk = 0.5f;
        long long vprev = 0;
        // start the task at offset q (skipping padding kernels of a partial block): unit q / KB
        // (a tree, or a tree's clock sub-range), kernel q % KB.  A sub-range [lo, end) walks from
        // the root at clock lo and, at its end, takes its last value back out at D[end] so the
        // difference arrays stay exact.  Returns false when the lane's tasks are exhausted.
        auto start = [&]() {
            while (q < seg1 && (q & (KB - 1)) >= nvalid) q = t.dyn ? atomicAdd(&s_pool[lane], 32) : q + NT;
            if (q >= seg1) return false;
            const int kk = q & (KB - 1);
            xb = xs_a + 4u * (unsigned)kk;
            const int ts = q >> KBL;
            int2 un = make_int2(ts, 0);
            if (SUB) un = units[ts];
            const int tti = un.x;
            const TmTree tr = stree[tti];
            bk = tr.root;
            blocks = tr.blocks;
            drow = dk + (size_t)kk * row + tr.slot_off;
            if (!FXALL) {
                const int mi = smodel[tti];
                fxm = s_fx[mi] != 0;                                         // as k_cut_blocks converted them
                scale = s_scale[mi];
            }
            if (SUB) {
                lo = un.y & 0xffff;
                end = un.y >> 16;
            }
            clk = (float)lo + 0.5f;                                          // clock lo enters as lo + 0.5
            tmin = CUDART_INF_F;
            sn = 0;
            vprev = 0;
            return true;
        };
        bool active = start();
        while (active) {                                                     // lanes leave as they finish
            uint4 A, B;
            const int cur = bk;
            ldg_blk256(blocks + 2 * (size_t)cur, A, B);
            float cb;
            bool at_leaf;
            const unsigned g = tm_step(A, B, xb, rs, clk, cb, at_leaf);
            bk = (int)g;
            if (cb < tmin) {                                                 // new record
                if (sn < kTmS) {                                             // deeper ones are not kept:
                    sts_u(sb_a + kEnt * (unsigned)sn, (unsigned)cur);        // resuming at an ancestor on
                    sts_f(sc_a + kEnt * (unsigned)sn, cb);                   // the path is still exact
                    ++sn;
                }
                tmin = cb;
            }
            if (at_leaf) {
                // run [lo, hi): hi = smallest left-turn cut; D[lo] += v - v_prev (exact int64)
                const int hi = tmin < CUDART_INF_F ? (int)tmin : n_f;
                const long long v = (FXALL || fxm) ? (long long)(int)g
                                                   : __double2ll_rn(__dmul_rn((double)__uint_as_float(g), scale));
                atomicAdd(reinterpret_cast<unsigned long long*>(drow + lo), (unsigned long long)(v - vprev));
                vprev = v;
                if (hi < end) {
                    // resume at the deepest kept record's block (popped); the next one is the bound
                    --sn;
                    bk = (int)lds_u(sb_a + kEnt * (unsigned)sn);
                    tmin = sn > 0 ? lds_f(sc_a + kEnt * (unsigned)(sn - 1)) : CUDART_INF_F;
                    lo = hi;
                    clk = (float)hi + 0.5f;
                } else {
                    if (SUB && end < n_f)                                    // sub-range end: D[end] -= v
                        atomicAdd(reinterpret_cast<unsigned long long*>(drow + end), (unsigned long long)(-v));
                    q = t.dyn ? atomicAdd(&s_pool[lane], 32) : q + NT;
                    if (!SUB) lo = 0;
                    active = start();
                }
            }
        }
        s0 = s1;
    }
}

// Clock-specialised copy of a model's 2-level blocks (see the header and kClkN above): every
// clock-split threshold (code == F) becomes its cut index #{i : f_i <= thr} as an fp32 integer,
// leaves become int32 fixed point when the model allows, clock splits are flagged and leaves are
// folded into grandchild slots.  One thread per block.
__global__ void __launch_bounds__(256) k_cut_blocks(const uint4* __restrict__ in, long long n_blocks, int F,
                                                    const float* __restrict__ freqs, int n_f,
                                                    double fx_scale, uint4* __restrict__ out) {
    const long long b = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= n_blocks) return;
    uint4 A = in[2 * b];
    const uint4 B = in[2 * b + 1];
    unsigned w[3] = {A.x, A.y, A.z};
    unsigned g[4] = {B.x, B.y, B.z, B.w};
    int code[3];
#pragma unroll
    for (int q = 0; q < 3; ++q) {
        code[q] = (int)((A.w >> (8 * q)) & 0xffu);
        if (code[q] > F && fx_scale != 0.0) {
            // leaf value (one-leaf tree at q = 0, child leaf at q = 1, 2) -> int32 v * 2^s, exact
            w[q] = (unsigned)__double2int_rn(__dmul_rn((double)__uint_as_float(w[q]), fx_scale));
            continue;
        }
        if (code[q] != F) continue;
        const float thr = __uint_as_float(w[q]);
        int l = 0, h = n_f;                                  // #{i : f_i <= thr}
        while (l < h) {
            const int mid = (l + h) >> 1;
            if (__ldg(freqs + mid) <= thr) l = mid + 1; else h = mid;
        }
        w[q] = __float_as_uint((float)l);
    }
    unsigned lm = (A.w >> 24) & 0xfu;
    if (fx_scale != 0.0) {
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if ((lm >> q) & 1u) g[q] = (unsigned)__double2int_rn(__dmul_rn((double)__uint_as_float(g[q]), fx_scale));
    }
    if (code[0] > F) {                                       // one-leaf tree
        code[1] = code[2] = F + 1;
        g[0] = g[1] = g[2] = g[3] = w[0];
        lm = 0xfu;
    } else {
        if (code[1] > F) { g[0] = g[1] = w[1]; lm |= 3u; }
        if (code[2] > F) { g[2] = g[3] = w[2]; lm |= 12u; }
    }
    A.x = w[0];
    A.y = w[1];
    A.z = w[2];
    A.w = (unsigned)code[0] | ((unsigned)code[1] << 8) | ((unsigned)code[2] << 16) | (lm << 24) |
          (code[0] == F ? kClkN : 0u) | (code[1] == F ? kClkC0 : 0u) | (code[2] == F ? kClkC1 : 0u);
    out[2 * b] = A;
    out[2 * b + 1] = make_uint4(g[0], g[1], g[2], g[3]);
}

// Shared-memory layout of a finish tile of KT kernels: fp64 and fp32 outputs per (model, kernel,
// clock), the clock table, the kernels' features (stride XS) and the exact sums [KT][nslot][n_f].
struct TmFinishSmem {
    double* mv0;     // [NM][KT][n_f]
    float* sv0;      // [NM][KT][n_f]
    float* fr;       // [n_f]
    float* xk;       // [KT][XS]
    long long* sD;   // [KT][nslot][n_f], 16-byte aligned
};
__device__ __forceinline__ TmFinishSmem tm_finish_layout(unsigned char* smem, int NM, int KT, int n_f, int XS) {
    TmFinishSmem L;
    L.mv0 = reinterpret_cast<double*>(smem);
    L.sv0 = reinterpret_cast<float*>(L.mv0 + (size_t)NM * KT * n_f);
    L.fr = L.sv0 + (size_t)NM * KT * n_f;
    L.xk = L.fr + n_f;
    L.sD = reinterpret_cast<long long*>(L.xk + KT * XS + 1);
    L.sD = reinterpret_cast<long long*>((reinterpret_cast<uintptr_t>(L.sD) + 15) & ~(uintptr_t)15);
    return L;
}

// The finish of nk kernels (k0 = global index of the first) whose exact leaf sums per (kernel,
// slot, clock) sit in L.sD: as difference arrays (scan: exact prefix sums first, in place) or as
// the sums themselves.  Forest mean and linear member per (model, clock) (combine), then
// finish_tile4 (SVR members, normalisation, selection).  Whole CTA; the caller has synchronised.
__device__ __forceinline__ void tm_finish_tile(const TmArgs& t, const TmFinishSmem& L, int KT, int nk, long long k0,
                                               bool scan) {
    const SweepArgs& a = t.s;
    const int n_f = a.n_f, F = a.F, XS = a.xs, NM = t.nm;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (int p = warp; p < NM * nk; p += nw) {                                // p = kernel * NM + model
        const int pk = p / NM, pm = p - pk * NM;
        if (pm >= 2 && !a.has_x[pm - 2]) continue;
        const DevModel& m = model_of(a, pm);
        double* out = L.mv0 + ((size_t)pm * KT + pk) * n_f;
        const float* xrow = L.xk + pk * XS;
        const int slot = t.slot_of[pm];
        const double lin_s = linear_static(m, xrow, F);                     // once per (kernel, model)
        if (slot < 0) {
            for (int i = lane; i < n_f; i += 32) out[i] = combine_pre(m, 0.0, lin_s, L.fr[i], F);
            continue;
        }
        long long* Dm = L.sD + ((size_t)pk * t.nslot + slot) * n_f;
        if (scan) {
            const int chunk = (n_f + 31) / 32;
            const int i0 = min(n_f, lane * chunk), i1 = min(n_f, i0 + chunk);
            long long run = 0;
            for (int i = i0; i < i1; ++i) run += Dm[i];
            long long excl = run;                                             // inclusive scan of chunk sums
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const long long y = __shfl_up_sync(0xffffffffu, excl, off);
                if (lane >= off) excl += y;
            }
            excl -= run;
            for (int i = i0; i < i1; ++i) {                                   // exact prefix sums in place
                excl += Dm[i];
                Dm[i] = excl;
            }
            __syncwarp();
        }
        // every clock independently (lane-strided, unrolled: the fp64 chains overlap)
        const double inv = m.fx_inv;
#pragma unroll 4
        for (int i = lane; i < n_f; i += 32) {
            const double forest_sum = __dmul_rn(__ll2double_rn(Dm[i]), inv);  // RN(exact sum)
            out[i] = combine_pre(m, forest_sum, lin_s, L.fr[i], F);
        }
    }
    __syncthreads();
    double* mv[4];
    float* sv[4];
    for (int m = 0; m < 4; ++m) {
        const bool present = m < 2 || (NM > 2 && a.has_x[m - 2]);
        mv[m] = present ? L.mv0 + (size_t)m * KT * n_f : nullptr;
        sv[m] = present ? L.sv0 + (size_t)m * KT * n_f : nullptr;
    }
    finish_tile4(a, mv, sv, nk, k0);
}

// Finish of KT kernels per CTA after k_tm_walk: stage and zero the D rows, exact prefix sums,
// then tm_finish_tile.
__global__ void __launch_bounds__(256) k_tm_finish(const __grid_constant__ TmArgs t) {
    const SweepArgs& a = t.s;
    extern __shared__ __align__(16) unsigned char smem[];
    const int n_f = a.n_f, F = a.F, KT = a.tile_k, XS = a.xs;
    const int k0s = blockIdx.x * KT;
    const int nk = min(KT, t.nks - k0s);
    const long long k0 = t.slab0 + k0s;
    const TmFinishSmem L = tm_finish_layout(smem, t.nm, KT, n_f, XS);
    const float* gfeat = a.features + k0 * F;
    for (int e = threadIdx.x; e < nk * F; e += blockDim.x) {
        const int r = e / F;
        L.xk[r * XS + (e - r * F)] = __ldg(gfeat + e);
    }
    for (int i = threadIdx.x; i < n_f; i += blockDim.x) L.fr[i] = __ldg(a.freqs + i);
    // launched as a programmatic dependent of k_tm_walk (same stream): everything above overlaps
    // the walk's tail; D is read only after the walk grid has completed (no-op otherwise)
    asm volatile("griddepcontrol.wait;" ::: "memory");
    // this CTA's D rows are one contiguous region: stage it with independent coalesced loads,
    // then zero it for the next call
    long long* gD = t.D + (size_t)k0s * t.nslot * n_f;
    const int nd = nk * t.nslot * n_f;
    for (int e = threadIdx.x; e < nd; e += blockDim.x) L.sD[e] = __ldcg(gD + e);
    __syncthreads();
    for (int e = threadIdx.x; e < nd; e += blockDim.x) gD[e] = 0;
    tm_finish_tile(t, L, KT, nk, k0, true);
}

// Single-launch path for small batches: one CTA per kernel walks every (tree,
// clock) pair directly from the root on the clock-cut blocks (clock i enters as i + 0.5, as in
// k_tm_walk), adds the leaf's exact fixed-point value into the kernel's int64 sums in shared
// memory (order-free), then runs the finish in the same CTA: no difference arrays, no second
// launch.  STAGE: the call's clock-cut blocks fit in shared memory and are copied there first
// (coalesced 16-byte loads, all independent), so the walks' dependent block fetches cost shared-
// memory latency instead of L2 / DRAM latency.
template <bool FXALL, bool STAGE>
__global__ void __launch_bounds__(512, 1) k_tm_small(const __grid_constant__ TmArgs t) {
    const SweepArgs& a = t.s;
    extern __shared__ __align__(16) unsigned char smem[];
    const int n_f = a.n_f, F = a.F, XS = a.xs;
    const long long k0 = t.slab0 + blockIdx.x;
    const TmFinishSmem L = tm_finish_layout(smem, t.nm, 1, n_f, XS);
    float* xw = reinterpret_cast<float*>(L.sD + (size_t)t.nslot * n_f);      // [F + 2] walk features
    uint4* sblk = reinterpret_cast<uint4*>((reinterpret_cast<uintptr_t>(xw + F + 2) + 15) & ~(uintptr_t)15);
    __shared__ int s_fx[4];
    __shared__ double s_scale[4];
    __shared__ const uint4* s_blocks[4];                                      // per model: its blocks
    const int T0 = trees_of(a, 0), T1 = trees_of(a, 1), T2 = t.nm > 2 ? trees_of(a, 2) : 0;
    const int c1 = T0, c2 = c1 + T1, c3 = c2 + T2, TT = c3 + (t.nm > 2 ? trees_of(a, 3) : 0);
    if (threadIdx.x == 0) {
        size_t off = 0;                                                       // staged: uint4 offset
        for (int m = 0; m < 4; ++m) {
            if (!trees_of(a, m)) continue;
            const DevModel& d = model_of(a, m);
            s_fx[m] = d.fx32;
            s_scale[m] = d.fx_scale;
            s_blocks[m] = STAGE ? sblk + off : d.blocks;
            off += 2 * (size_t)d.nblk;
        }
    }
    if (STAGE) {                                                              // every model's blocks, in order
        size_t off = 0;
        for (int m = 0; m < 4; ++m) {
            if (!trees_of(a, m)) continue;
            const DevModel& d = model_of(a, m);
            const int n16 = 2 * d.nblk;
            for (int e = threadIdx.x; e < n16; e += blockDim.x) sblk[off + e] = __ldg(d.blocks + e);
            off += n16;
        }
    }
    const float* gfeat = a.features + k0 * F;
    for (int e = threadIdx.x; e < F; e += blockDim.x) {
        const float v = __ldg(gfeat + e);
        L.xk[e] = v;
        xw[e] = v;
    }
    if (threadIdx.x < 2) xw[F + threadIdx.x] = 0.0f;                          // row F unused, F + 1 = 0
    for (int i = threadIdx.x; i < n_f; i += blockDim.x) L.fr[i] = __ldg(a.freqs + i);
    for (int e = threadIdx.x; e < t.nslot * n_f; e += blockDim.x) L.sD[e] = 0;
    __syncthreads();
    const unsigned xs_a = su32(xw);
    const int nw = TT * n_f;
    for (int w = threadIdx.x; w < nw; w += blockDim.x) {
        const int tree = w / n_f, i = w - tree * n_f;
        const int mi = tree < c1 ? 0 : tree < c2 ? 1 : tree < c3 ? 2 : 3;
        const DevModel& d = model_of(a, mi);
        const uint4* blocks = s_blocks[mi];
        int bk = __ldg(d.broot + (tree - (mi == 0 ? 0 : mi == 1 ? c1 : mi == 2 ? c2 : c3)));
        const float clk = (float)i + 0.5f;
        while (true) {
            uint4 A, B;
            if (STAGE) {
                A = blocks[2 * (size_t)bk];
                B = blocks[2 * (size_t)bk + 1];
            } else {
                ldg_blk256(blocks + 2 * (size_t)bk, A, B);
            }
            float cb;
            bool at_leaf;
            const unsigned g = tm_step(A, B, xs_a, 4u, clk, cb, at_leaf);
            if (at_leaf) {
                const long long v = (FXALL || s_fx[mi]) ? (long long)(int)g
                                                        : __double2ll_rn(__dmul_rn((double)__uint_as_float(g), s_scale[mi]));
                atomicAdd(reinterpret_cast<unsigned long long*>(L.sD + (size_t)t.slot_of[mi] * n_f + i),
                          (unsigned long long)v);
                break;
            }
            bk = (int)g;
        }
    }
    __syncthreads();
    tm_finish_tile(t, L, 1, 1, k0, false);
}

}  // namespace syn

