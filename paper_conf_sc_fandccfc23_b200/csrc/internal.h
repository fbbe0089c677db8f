// internal.h — device-side data layout shared by the C-ABI host code and the kernels.
// Not part of the public ABI (include/synergy.h).  See DESIGN.md "Data layout in HBM".
#pragma once
#include <cstdint>

namespace syn {

// Packed forest node, 8 bytes, breadth-first per tree with the two children adjacent
// (k_gen_forest's direct walks):
//   .x = bits of the fp32 threshold (internal) or leaf value (leaf)
//   .y = meta = (delta << 8) | code,  delta signed 24-bit
//        code in [0, F)  : split on static feature `code`
//        code == F       : split on the core clock (input F)
//        code == F + 1   : leaf
//   next = idx + delta + (x <= thr ? 0 : 1)
constexpr int kCodeBits = 8;
constexpr int kMaxDelta = (1 << 23) - 1;

struct DevModel {
    const uint2* nodes;      // [n_nodes]
    const int2* trees;       // [n_trees] {first node (BFS root), depth}
    const double* lin_w;     // [n_inputs]
    double lin_b;
    double lin_weight;       // 0 => absent
    double forest_weight;    // 0 => absent
    int n_trees;
    int depth;               // deepest root-to-leaf path over all trees (edges)
    // 2-level block layout (32 B per block, two uint4): words
    //   0: thr(n)  1: thr(c0)  2: thr(c1)  3: code(n) | code(c0) << 8 | code(c1) << 16 |
    //                                         leafmask << 24 (grandchild slot holds a leaf value)
    //   4..7: grandchild slots g = 2*d0 + d1: block index, or fp32 leaf-value bits (leafmask)
    // A child c_d that is itself a leaf has code F+1 and its value in thr(c_d); a one-leaf tree
    // has code(n) = F+1.  Blocks exist for the root and every internal node at even depth, so
    // a root-to-leaf walk of depth D takes max(1, ceil(D / 2)) block loads.
    const uint4* blocks;
    const int* broot;        // [n_trees] root block of each tree
    const int* broot_lpt;    // [n_trees] the same roots in expected-cost order, alternating the
                             // costliest and the cheapest remaining tree (small batches, see run_tm)
    // per-tree clock sub-range split for small batches (k_tm_walk unit tables): {first unit of the
    // tree within the model, sub-ranges}; sub-ranges ~ ceil(expected runs / the model's mean), so
    // the longest (kernel, tree) walks are cut into pieces of about average length
    const int2* tsplit;      // [n_trees]
    int units_split;         // sum of the sub-ranges over the trees
    int nblk;                // blocks of all trees (tree t owns [broot[t], broot[t+1] or nblk))
    // exact leaf sums (Q8): every (finite) fp32 leaf v is an integer multiple of 2^-s
    // (s from the smallest leaf ulp).  fx_ok: n_trees * max|v| * 2^s < 2^62, so v * 2^s is an
    // exact int64 and int64 sums are exact in any order (k_tm_walk); otherwise k_gen_forest sums
    // v * 2^s exactly in a multi-word integer accumulator.
    int fx_ok;
    int fx32;                // fx_ok and every |v| * 2^s < 2^31 (int32 fixed-point leaves fit)
    int fx_s;                // s
    double fx_scale;         // 2^s
    double fx_inv;           // 2^-s
    // SVR_RBF member: svr = b + sum_j dual_j exp(-gamma ||(x - mean)/scale - sv_j||^2)
    double svr_weight;       // 0 => absent
    int n_sv;
    const float* sv;         // [n_sv][n_inputs]
    const double* dual;      // [n_sv]
    const double* in_mean;   // [n_inputs]
    const double* in_scale;  // [n_inputs]
    double svr_gamma, svr_b;
    int svr_eU;              // max_j |dual_j| < 2^svr_eU (k_svr_tc's digit scale)
    // per call (k_svr): svr_splits partial contractions over SV ranges, [svr_splits][n_k][n_f],
    // summed in split order (+ svr_b) by finish_tile
    const double* svr_p;
    int svr_splits;
};

// SVR contraction tiling (kernels_svr.cuh): 8 warps x kSvrRows kernels = kSvrTK kernels per CTA,
// 32 x CPT clocks, SVs staged kSvrJC at a time through a kSvrStages-deep bulk-copy ring
constexpr int kSvrRows = 8;
constexpr int kSvrTK = 8 * kSvrRows;
constexpr int kSvrJC = 16;
constexpr int kSvrStages = 3;
constexpr int kSvrMaxSplits = 16;

struct SvrArgs {
    const float* features;   // [n_k][F]
    long long n_k;
    int F;
    const float* freqs;      // [n_f]
    int n_f;
    const float* sv;         // [n_sv][F + 1]
    const double* dual;
    const double* in_mean;
    const double* in_scale;
    double gamma;
    int n_sv;
    int n_svp;               // n_sv rounded up to kSvrJC (padding rows are zero)
    int tn;                  // clock tile (32 * CPT)
    int chunks_per_split;    // kSvrJC-SV chunks per split (blockIdx.z)
    long long slab0;         // first kernel of this slab
    int nks;                 // kernels in this slab
    double* Ut;              // [ceil(nks / kSvrTK)][n_svp][kSvrTK]   U_kj = dual_j e^{-gamma A_kj}
    double* Vt;              // [ceil(n_f / tn)][n_svp][tn]           V_ji = e^{-gamma B_ji}
    double* P;               // [splits][n_k][n_f] partial contractions
};

constexpr int kMaxTargets = 16;

enum Mode : int { kModePredict = 0, kModeSweep = 1 };

struct SweepArgs {
    DevModel ms, me;         // speedup, energy
    DevModel mx[2];          // four-model variant: direct EDP, ED2P models
    int has_x[2];            // which of mx are present
    const float* features;   // [n_k][F]
    long long n_k;
    int F;                   // static features; clock is input F
    const float* freqs;      // [n_f]
    int n_f;
    int def;                 // default clock index; -1 = raw (predict only)
    int n_t;
    int kind[kMaxTargets];
    double frac[kMaxTargets];  // x / 100 (fp64, host: the oracle's division)
    int* choice;             // [n_k][n_t] (sweep)
    float* S_out;            // [n_k][n_f] or null
    float* E_out;
    float* X_out[2];         // direct EDP / ED2P normalised predictions, [n_k][n_f] or null
    int mode;
    int tile_k;              // kernels per finish CTA
    int xs;                  // x-vector stride in smem (floats)
};

struct SelectArgs {
    const float* S;
    const float* E;
    long long n_k;
    int n_f;
    int def;
    int n_t;
    int kind[kMaxTargets];
    double frac[kMaxTargets];  // x / 100 (fp64, host: the oracle's division)
    int* choice;
};

}  // namespace syn
