// kernels_svr_tc.cuh — SVR_RBF contraction P = U V on the 5th-generation tensor cores (tcgen05).
//
// The SVR member over a clock sweep is the contraction P[k][i] = sum_j U[k][j] V[j][i] with
// U[k][j] = dual_j e^{-gamma A_kj} (any sign) and V[j][i] = e^{-gamma B_ji} (Q24,
// kernels_svr.cuh).  tcgen05 has no fp64 kind, and the duals cancel (sum_j |U V| reaches ~130x
// |prediction| on the bench model), so a TF32/BF16 split with fp32 accumulation cannot hold the
// 1e-5 bar.  This path uses exact integer tensor-core products instead (an Ozaki-style split):
//
//   * every row k of U is scaled by 2^-eU_k (eU_k = the exponent of the row's largest |U|, so the
//     scaled row lies in (-1, 1)) and written as 7 signed 7-bit digits, x = sum_p d_p 2^-7(p+1),
//     |d_p| <= 127, truncating below 2^-49; every clock column i of V likewise with 2^-eV_i;
//   * U V = 2^(eU_k + eV_i) sum_{p,q} 2^-7(p+q+2) (D_p E_q), and each digit product D_p E_q is an
//     int8 x int8 GEMM with exact int32 accumulation (tcgen05.mma kind::i8: |sum| <= 127^2 * 512 *
//     7 < 2^31).  Products of equal level L = p + q share one TMEM accumulator; levels L >= 7 are
//     dropped (the 28 products with L <= 6 are kept);
//   * the epilogue reads the 7 level accumulators (tcgen05.ld), sums 2^-7(L+2) acc_L in fp64 and
//     scales by 2^(eU + eV).  The value differs from the exact contraction by at most about
//     n_sv * 2^-46 * max_j|U_kj| * max_j V_ji (digit truncation and dropped levels), far inside
//     the 1e-5 bar (tests/test_gpu_svr.py compares with the oracle and with the fp64 k_svr path).
//
// Tiles: 128 kernels x 64 clocks per CTA (one M=128, N=64 MMA shape), SVs in chunks of 64 (two
// K=32 MMAs per digit pair per chunk).  Operands are pre-laid by k_svr_quant in the canonical
// K-major, no-swizzle UMMA layout (8-row x 16-byte core matrices: LBO = 128 B between K-adjacent
// core matrices, SBO = 512 B between 8-row groups), all 7 digit planes of a (tile, chunk) in one
// contiguous block, so each chunk arrives by one 1-D bulk copy per operand (cp.async.bulk, the TMA
// engine) into a 2-stage mbarrier ring.  Warp roles: warp 0 producer, warp 1 TMEM allocation and
// MMA issue (one elected lane), warps 2-5 epilogue (TMEM lane quarters).  The SV range may be split
// across CTAs (blockIdx.z); each split writes its partial plane P[z], which the finish sums in
// split order (add_svr_unit), exactly as for k_svr.
#pragma once
#include "kernels_svr.cuh"

namespace syn {

constexpr int kTcM = 128, kTcN = 64, kTcKC = 64, kTcDig = 7, kTcStages = 2;
constexpr unsigned kTcABytes = (unsigned)kTcDig * kTcM * kTcKC;   // one chunk of U, all digit planes
constexpr unsigned kTcBBytes = (unsigned)kTcDig * kTcN * kTcKC;   // one chunk of V
constexpr int kTcThreads = 192;
constexpr size_t kTcSmem = (size_t)kTcStages * (kTcABytes + kTcBBytes) + 256;

struct SvrTcArgs {
    const double* src;       // k_svr_quant: [rows / 64][n_svp][64] fp64 (Ut or Vt tiles)
    int rows;                // k_svr_quant: rows of the source (kernels of the slab, or clocks)
    int tile_rows;           // k_svr_quant: rows per destination tile (kTcM for U, kTcN for V)
    unsigned char* dst;      // k_svr_quant: [tiles][n_chunks][kTcDig][tile_rows x kTcKC] int8
    int* ex;                 // [rows] exponents (k_svr_quant writes, k_svr_tc reads)
    int n_svp;               // SVs, padded to a multiple of kTcKC
    // k_svr_tc
    const unsigned char* Uq;
    const unsigned char* Vq;
    const int* eU;
    const int* eV;
    double* P;               // [splits][n_k][n_f]
    long long slab0, n_k;
    int nks, n_f;
    int chunks_per_split;
};

// Byte offset of element (row r, K byte kb) inside one digit plane of a tile (canonical K-major,
// no swizzle): core matrix (r / 8, kb / 16) at (r / 8) * SBO + (kb / 16) * LBO, 16-byte rows.
__device__ __forceinline__ unsigned tc_off(int r, int kb) {
    return (unsigned)((r >> 3) * 512 + (kb >> 4) * 128 + (r & 7) * 16 + (kb & 15));
}

// Exponent of each source row's largest |value| (x < 2^e for all x of the row); one thread per row.
__global__ void __launch_bounds__(256) k_svr_rowexp(const __grid_constant__ SvrTcArgs a) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= a.rows) return;
    const double* s = a.src + (size_t)(r >> 6) * a.n_svp * 64 + (r & 63);
    double m = 0.0;
    for (int j = 0; j < a.n_svp; ++j) m = fmax(m, fabs(__ldg(s + (size_t)j * 64)));
    int e = 0;
    if (m > 0.0) frexp(m, &e);                                   // m in [2^(e-1), 2^e)
    a.ex[r] = e;
}

// Digit planes: thread per (row, 16 consecutive SVs) writes one 16-byte row segment per digit.
__global__ void __launch_bounds__(256) k_svr_quant(const __grid_constant__ SvrTcArgs a) {
    const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const int groups = a.n_svp / 16;
    const int tiles = (a.rows + a.tile_rows - 1) / a.tile_rows;
    if (t >= (long long)tiles * a.tile_rows * groups) return;
    const int g = (int)(t % groups);
    const int rr = (int)(t / groups);                            // row over padded tiles
    const int tile = rr / a.tile_rows, r = rr - tile * a.tile_rows;
    const int j0 = g * 16;
    const int chunk = j0 / kTcKC, kb = j0 % kTcKC;
    const int n_chunks = a.n_svp / kTcKC;
    unsigned w[kTcDig][4];
#pragma unroll
    for (int p = 0; p < kTcDig; ++p) w[p][0] = w[p][1] = w[p][2] = w[p][3] = 0u;
    if (rr < a.rows) {
        const int e = a.ex[rr];
        const double* s = a.src + (size_t)(rr >> 6) * a.n_svp * 64 + (rr & 63);
#pragma unroll 4
        for (int q = 0; q < 16; ++q) {
            double x = scalbn(__ldg(s + (size_t)(j0 + q) * 64), -e);      // |x| < 1 (exact unless it
                                                                          // underflows: < 2^-1074 of the max)
#pragma unroll
            for (int p = 0; p < kTcDig; ++p) {
                x = __dmul_rn(x, 128.0);                           // exact
                const double d = trunc(x);                         // |d| <= 127
                x = __dsub_rn(x, d);                               // exact
                const unsigned byte = (unsigned)(int)d & 0xffu;
                w[p][q >> 2] |= byte << (8 * (q & 3));
            }
        }
    }
    unsigned char* base = a.dst + ((size_t)tile * n_chunks + chunk) * kTcDig * a.tile_rows * kTcKC;
#pragma unroll
    for (int p = 0; p < kTcDig; ++p)
        *reinterpret_cast<uint4*>(base + (size_t)p * a.tile_rows * kTcKC + tc_off(r, kb)) =
            make_uint4(w[p][0], w[p][1], w[p][2], w[p][3]);
}

__device__ __forceinline__ unsigned long long tc_desc(unsigned saddr) {
    return (unsigned long long)((saddr >> 4) & 0x3FFFu) | (8ull << 16) | (32ull << 32) | (1ull << 46);
}

// tcgen05.mma kind::i8 instruction descriptor: s32 accumulator, signed int8 A and B, both K-major,
// M = 128, N = 64.
constexpr unsigned kTcIdesc = (2u << 4) | (1u << 7) | (1u << 10) | ((unsigned)(kTcN >> 3) << 17) |
                              ((unsigned)(kTcM >> 4) << 24);

__global__ void __launch_bounds__(kTcThreads, 1) k_svr_tc(const __grid_constant__ SvrTcArgs a) {
    extern __shared__ __align__(128) unsigned char tcs[];
    unsigned char* As = tcs;                                             // [stages][A chunk]
    unsigned char* Bs = tcs + (size_t)kTcStages * kTcABytes;             // [stages][B chunk]
    unsigned long long* full = reinterpret_cast<unsigned long long*>(Bs + (size_t)kTcStages * kTcBBytes);
    unsigned long long* empty = full + kTcStages;
    unsigned long long* accb = empty + kTcStages;
    unsigned* tmem_slot = reinterpret_cast<unsigned*>(accb + 1);
    const int mt = blockIdx.x, nt = blockIdx.y;
    const int n_chunks = a.n_svp / kTcKC;
    const int c0 = blockIdx.z * a.chunks_per_split;
    const int nch = min(a.chunks_per_split, n_chunks - c0);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kTcStages; ++s) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, 1);
        }
        mbar_init(accb, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 1) {                                                     // 512 TMEM columns: 7 x 64 used
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;"
                     :: "r"(svr_su32(tmem_slot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const unsigned tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {                                                 // producer
            const unsigned char* ug = a.Uq + ((size_t)mt * n_chunks + c0) * kTcABytes;
            const unsigned char* vg = a.Vq + ((size_t)nt * n_chunks + c0) * kTcBBytes;
            for (int c = 0; c < nch; ++c) {
                const int s = c % kTcStages;
                if (c >= kTcStages) mbar_wait(empty + s, (unsigned)(((c / kTcStages) - 1) & 1));
                mbar_expect_tx(full + s, kTcABytes + kTcBBytes);
                bulk_g2s(As + (size_t)s * kTcABytes, ug + (size_t)c * kTcABytes, kTcABytes, full + s);
                bulk_g2s(Bs + (size_t)s * kTcBBytes, vg + (size_t)c * kTcBBytes, kTcBBytes, full + s);
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {                                                 // MMA issue
            for (int c = 0; c < nch; ++c) {
                const int s = c % kTcStages;
                mbar_wait(full + s, (unsigned)((c / kTcStages) & 1));
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const unsigned abase = svr_su32(As + (size_t)s * kTcABytes);
                const unsigned bbase = svr_su32(Bs + (size_t)s * kTcBBytes);
#pragma unroll 1
                for (int p = 0; p < kTcDig; ++p) {
#pragma unroll 1
                    for (int q = 0; p + q < kTcDig; ++q) {
                        const unsigned d = tmem + (unsigned)((p + q) * kTcN);
#pragma unroll
                        for (int kk = 0; kk < kTcKC / 32; ++kk) {
                            const unsigned long long ad = tc_desc(abase + (unsigned)(p * kTcM * kTcKC + kk * 256));
                            const unsigned long long bd = tc_desc(bbase + (unsigned)(q * kTcN * kTcKC + kk * 256));
                            const unsigned acc = (c > 0 || p > 0 || kk > 0) ? 1u : 0u;   // first write of level p+q
                            asm volatile(
                                "{\n\t.reg .pred pa;\n\t"
                                "setp.ne.b32 pa, %4, 0;\n\t"
                                "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, {%5, %5, %5, %5}, pa;\n\t}"
                                :: "r"(d), "l"(ad), "l"(bd), "r"(kTcIdesc), "r"(acc), "r"(0u) : "memory");
                        }
                    }
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                             :: "r"(svr_su32(empty + s)) : "memory");
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         :: "r"(svr_su32(accb)) : "memory");
        }
    } else {                                                             // epilogue: warps 2..5
        const int quarter = warp & 3;                                    // TMEM lanes 32 * quarter ..
        const int r = quarter * 32 + lane;                               // row of the tile (kernel)
        mbar_wait(accb, 0u);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const long long k = (long long)mt * kTcM + r;                   // slab-relative kernel
        const bool rv = k < a.nks;
        const int eu = rv ? __ldg(a.eU + k) : 0;
        double* P = a.P + (size_t)blockIdx.z * a.n_k * a.n_f + (size_t)(a.slab0 + k) * a.n_f;
#pragma unroll 1
        for (int cb = 0; cb < kTcN / 16; ++cb) {
            double s[16];
#pragma unroll
            for (int c = 0; c < 16; ++c) s[c] = 0.0;
#pragma unroll 1
            for (int L = 0; L < kTcDig; ++L) {
                unsigned v[16];
                const unsigned taddr = tmem + ((unsigned)(quarter * 32) << 16) + (unsigned)(L * kTcN + cb * 16);
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
                    "%12, %13, %14, %15}, [%16];"
                    : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
                      "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
                      "=r"(v[14]), "=r"(v[15])
                    : "r"(taddr));
                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                const double w = scalbn(1.0, -7 * (L + 2));                        // 2^-7(L+2)
#pragma unroll
                for (int c = 0; c < 16; ++c) s[c] = __fma_rn((double)(int)v[c], w, s[c]);   // exact products
            }
            if (rv) {
#pragma unroll
                for (int c = 0; c < 16; ++c) {
                    const int i = nt * kTcN + cb * 16 + c;
                    if (i < a.n_f) P[i] = scalbn(s[c], eu + __ldg(a.eV + i));
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tmem) : "memory");
}

}  // namespace syn
