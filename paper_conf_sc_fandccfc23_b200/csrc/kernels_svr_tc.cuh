// kernels_svr_tc.cuh — SVR_RBF contraction P = U V on the 5th-generation tensor cores (tcgen05).
//
// The SVR member over a clock sweep is the contraction P[k][i] = sum_j U[k][j] V[j][i] with
// U[k][j] = dual_j e^{-gamma A_kj} (any sign) and V[j][i] = e^{-gamma B_ji} in (0, 1] (DESIGN.md
// Q24, kernels_svr.cuh).  tcgen05 has no fp64 kind, and the duals cancel (sum_j |U V| reaches
// ~130x |prediction| on the bench model), so a TF32/BF16 split with fp32 accumulation cannot hold
// the 1e-5 bar.  This path uses exact integer tensor-core products instead (an Ozaki-style split):
//
//   * U is scaled by 2^-eU (eU = the exponent of max_j |dual_j|, fixed per model: |U| <= max|dual|
//     < 2^eU) and V by 2^-1 (V <= 1 < 2^1), so both lie in (-1, 1); each scaled value x becomes the
//     integer X = round(x 2^54) written with 7 balanced base-256 digits, X = sum_p d_p 256^(6-p),
//     d_p in [-128, 127] (signed bytes), |x - X 2^-54| <= 2^-55;
//   * U V = 2^(eU + 1 - 108) sum_{p,q} 256^(12-p-q) (D_p E_q), and each digit product D_p E_q is an
//     int8 x int8 GEMM with exact int32 accumulation (tcgen05.mma kind::i8; |sum| <= 128^2 * n_sv
//     * 7 < 2^31 for n_sv <= 16384).  Products of equal level L = p + q share one TMEM accumulator
//     (7 levels x 32 columns); levels L >= 7 are dropped (the 28 pairs with L <= 6 are kept);
//   * the epilogue reads the 7 level accumulators (tcgen05.ld), sums 2^-(8L+12) acc_L in fp64 and
//     scales by 2^(eU + 1).  Digit rounding and the dropped levels change each term by at most
//     about 2^-53 max_j|dual_j| (both factors' scales are powers of two), so the value is within
//     n_sv 2^-53 max_j|dual_j| of the exact contraction — the same order as the fp64 path's
//     rounding bound (Q24) — and tests/test_gpu_svr.py compares it with the oracle and
//     with the fp64 k_svr reference (fp32 predictions equal or one ulp apart).
//
// Digits are produced where U and V are computed (k_svr_udig, k_svr_vdig), directly in the
// canonical K-major, no-swizzle UMMA layout (8-row x 16-byte core matrices; LBO = 128 B between the
// two K-adjacent core matrices of a 32-SV chunk, SBO = 256 B between 8-row groups), all 8 digit
// planes of a (tile, chunk) contiguous, so each chunk reaches shared memory by one 1-D bulk copy per
// operand (cp.async.bulk, the TMA engine) into a 3-stage mbarrier ring.  k_svr_tc: 128 kernels x 32
// clocks per CTA (M = 128, N = 32, K = 32 per MMA), two CTAs per SM (105 KB of shared memory and
// 256 TMEM columns each), so one CTA's MMAs overlap the other's epilogue and operand loads (the
// N = 64, one-CTA-per-SM version took 0.36 ms per c3 slab, this one 0.30); warp 0 producer, warp
// 1 TMEM allocation and MMA issue (one elected lane, 28 MMAs per chunk), warps 2-5 epilogue (TMEM
// lane quarters).  The SV
// range may be split across CTAs (blockIdx.z); each split writes its partial plane P[z], which the
// finish sums in split order (add_svr_unit), exactly as for k_svr.
#pragma once
#include "kernels_svr.cuh"

namespace syn {

constexpr int kTcM = 128, kTcN = 32, kTcKC = 32, kTcDig = 7, kTcStages = 3;
constexpr unsigned kTcAPlane = (unsigned)kTcM * kTcKC, kTcBPlane = (unsigned)kTcN * kTcKC;
constexpr unsigned kTcABytes = kTcDig * kTcAPlane;   // one 32-SV chunk of U, all digit planes
constexpr unsigned kTcBBytes = kTcDig * kTcBPlane;   // one chunk of V
constexpr int kTcThreads = 192;
constexpr int kTcCtasPerSm = 2;                      // 3-stage ring (105 KB) and 256 TMEM columns each
constexpr size_t kTcSmem = (size_t)kTcStages * (kTcABytes + kTcBBytes) + 256;

struct SvrTcArgs {
    SvrArgs s;               // features, clocks, SVs, duals, standardisation, gamma, slab
    unsigned char* Uq;       // [mtiles of the slab][n_chunks][kTcDig][128 x 32] int8
    unsigned char* Vq;       // [ntiles][n_chunks][kTcDig][kTcN x 32] int8
    int eU;                  // U scale exponent (max |dual| < 2^eU)
    int chunks_per_split;
};

// Byte offset of element (row r, SV kb within the chunk) inside one digit plane (canonical K-major,
// no swizzle): core matrix (r / 8, kb / 16) at (r / 8) * 256 + (kb / 16) * 128, 16-byte rows.
__device__ __forceinline__ unsigned tc_off(int r, int kb) {
    return (unsigned)((r >> 3) * 256 + (kb >> 4) * 128 + (r & 7) * 16 + (kb & 15));
}

// 16 consecutive values (x[q] in (-1, 1)) -> kTcDig digit planes, 16 bytes each, at base + p * plane.
// X = round(x 2^54) (an integer, |X| <= 2^54) is written in balanced base 256: the unique digits
// d_p in [-128, 127] with X = sum_p d_p 256^(kTcDig - 1 - p); |x - X 2^-54| <= 2^-55.  With
// C = 0x0080808080808080 (128 in each of the 7 digit positions), X + C is in [0, 256^7) and its
// base-256 digits are d_p + 128, so the signed bytes of (X + C) xor C are exactly the d_p (the
// digit-by-digit recurrence d = ((X + 128) mod 256) - 128, X = (X - d) / 256 gives the same digits).
__device__ __forceinline__ void tc_store_digits(const double (&x)[16], unsigned char* base, unsigned plane) {
    constexpr unsigned long long C = 0x0080808080808080ull;
    unsigned lo[16], hi[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) {
        const unsigned long long Z = ((unsigned long long)__double2ll_rn(scalbn(x[q], 54)) + C) ^ C;
        lo[q] = (unsigned)Z;
        hi[q] = (unsigned)(Z >> 32);
    }
#pragma unroll
    for (int p = 0; p < kTcDig; ++p) {
        const int bi = kTcDig - 1 - p;                                    // byte of Z holding d_p
        unsigned w[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const unsigned* h = bi < 4 ? lo : hi;
            const unsigned j = (unsigned)(bi & 3);
            const unsigned sel = j | ((4u + j) << 4);                    // [a_j, b_j] in bytes 0, 1
            const unsigned t1 = __byte_perm(h[4 * k], h[4 * k + 1], sel);
            const unsigned t2 = __byte_perm(h[4 * k + 2], h[4 * k + 3], sel);
            w[k] = __byte_perm(t1, t2, 0x5410u);                          // values 4k .. 4k+3
        }
        *reinterpret_cast<uint4*>(base + (size_t)p * plane) = make_uint4(w[0], w[1], w[2], w[3]);
    }
}

// U digits for a 128-kernel tile (blockIdx.x, slab-relative) and a 32-SV chunk (blockIdx.y):
// thread = (kernel r, 16-SV half h).  U_kj = dual_j exp(-gamma sum_{d<F} (z_kd - sv_jd)^2) in fp64
// (k_svr_u's arithmetic), scaled by 2^-eU.  Padding kernels / SVs are zero.
__global__ void __launch_bounds__(256) k_svr_udig(const __grid_constant__ SvrTcArgs t) {
    const SvrArgs& a = t.s;
    extern __shared__ __align__(16) double tz[];
    const int F = a.F;
    double* z = tz;                                                       // [128][F + 1]
    float* sv = reinterpret_cast<float*>(z + (size_t)kTcM * (F + 1));     // [32][F]
    const int mt = blockIdx.x, c = blockIdx.y;
    const long long kb = a.slab0 + (long long)mt * kTcM;
    const int nk = (int)min((long long)kTcM, a.slab0 + a.nks - kb);
    const int j0 = c * kTcKC;
    for (int e = threadIdx.x; e < kTcM * F; e += blockDim.x) {
        const int r = e / F, d = e - r * F;
        double v = 0.0;
        if (r < nk) v = __ddiv_rn(__dsub_rn((double)__ldg(a.features + kb * F + e), __ldg(a.in_mean + d)), __ldg(a.in_scale + d));
        z[r * (F + 1) + d] = v;
    }
    for (int e = threadIdx.x; e < kTcKC * F; e += blockDim.x) {
        const int q = e / F, d = e - q * F;
        sv[q * F + d] = j0 + q < a.n_sv ? __ldg(a.sv + (size_t)(j0 + q) * (F + 1) + d) : 0.0f;
    }
    __syncthreads();
    const int r = threadIdx.x >> 1, h = threadIdx.x & 1;
    double x[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) {
        const int j = j0 + 16 * h + q;
        double A = 0.0;
        for (int d = 0; d < F; ++d) {
            const double tt = __dsub_rn(z[r * (F + 1) + d], (double)sv[(16 * h + q) * F + d]);
            A = __dadd_rn(A, __dmul_rn(tt, tt));
        }
        x[q] = (r < nk && j < a.n_sv) ? scalbn(__dmul_rn(__ldg(a.dual + j), exp(-__dmul_rn(a.gamma, A))), -t.eU) : 0.0;
    }
    const int n_chunks = a.n_svp / kTcKC;
    tc_store_digits(x, t.Uq + ((size_t)mt * n_chunks + c) * kTcABytes + tc_off(r, 16 * h), kTcAPlane);
}

// V digits for a kTcN-clock tile (blockIdx.x) and a 32-SV chunk (blockIdx.y): thread = (clock r,
// 16-SV half h).  V_ji = exp(-gamma (z(f_i) - sv_jF)^2) (k_svr_v's arithmetic), scaled by 2^-1.
__global__ void __launch_bounds__(128) k_svr_vdig(const __grid_constant__ SvrTcArgs t) {
    const SvrArgs& a = t.s;
    const int nt = blockIdx.x, c = blockIdx.y;
    const int r = threadIdx.x >> 1, h = threadIdx.x & 1;
    const int i = nt * kTcN + r, F = a.F;
    double zc = 0.0;
    if (i < a.n_f) zc = __ddiv_rn(__dsub_rn((double)__ldg(a.freqs + i), __ldg(a.in_mean + F)), __ldg(a.in_scale + F));
    double x[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) {
        const int j = c * kTcKC + 16 * h + q;
        double v = 0.0;
        if (i < a.n_f && j < a.n_sv) {
            const double b = __dsub_rn(zc, (double)__ldg(a.sv + (size_t)j * (F + 1) + F));
            v = exp(-__dmul_rn(a.gamma, __dmul_rn(b, b)));
        }
        x[q] = __dmul_rn(v, 0.5);                                         // exact
    }
    const int n_chunks = a.n_svp / kTcKC;
    tc_store_digits(x, t.Vq + ((size_t)nt * n_chunks + c) * kTcBBytes + tc_off(r, 16 * h), kTcBPlane);
}

__device__ __forceinline__ unsigned long long tc_desc(unsigned saddr) {
    // start address >> 4 | LBO 128 B >> 4 | SBO 256 B >> 4 | descriptor version 1 (sm_100)
    return (unsigned long long)((saddr >> 4) & 0x3FFFu) | (8ull << 16) | (16ull << 32) | (1ull << 46);
}

// tcgen05.mma kind::i8 instruction descriptor: s32 accumulator, signed int8 A and B, both K-major,
// M = 128, N = kTcN.
constexpr unsigned kTcIdesc = (2u << 4) | (1u << 7) | (1u << 10) | ((unsigned)(kTcN >> 3) << 17) |
                              ((unsigned)(kTcM >> 4) << 24);

__global__ void __launch_bounds__(kTcThreads, kTcCtasPerSm) k_svr_tc(const __grid_constant__ SvrTcArgs t) {
    const SvrArgs& a = t.s;
    extern __shared__ __align__(128) unsigned char tcs[];
    unsigned char* As = tcs;                                             // [stages][A chunk]
    unsigned char* Bs = tcs + (size_t)kTcStages * kTcABytes;             // [stages][B chunk]
    unsigned long long* full = reinterpret_cast<unsigned long long*>(Bs + (size_t)kTcStages * kTcBBytes);
    unsigned long long* empty = full + kTcStages;
    unsigned long long* accb = empty + kTcStages;
    unsigned* tmem_slot = reinterpret_cast<unsigned*>(accb + 1);
    // clock tiles vary fastest across the grid, so the CTAs that share a kernel tile's U digits run
    // together and read them from DRAM once (L2 serves the others)
    const int nt = blockIdx.x, mt = blockIdx.y;
    const int n_chunks = a.n_svp / kTcKC;
    const int c0 = blockIdx.z * t.chunks_per_split;
    const int nch = min(t.chunks_per_split, n_chunks - c0);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kTcStages; ++s) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, 1);
        }
        mbar_init(accb, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 1) {                                                     // 256 TMEM columns: 7 x 32 used
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;"
                     :: "r"(svr_su32(tmem_slot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const unsigned tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {                                                 // producer
            const unsigned char* ug = t.Uq + ((size_t)mt * n_chunks + c0) * kTcABytes;
            const unsigned char* vg = t.Vq + ((size_t)nt * n_chunks + c0) * kTcBBytes;
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
                        const unsigned long long ad = tc_desc(abase + (unsigned)p * kTcAPlane);
                        const unsigned long long bd = tc_desc(bbase + (unsigned)q * kTcBPlane);
                        const unsigned acc = (c > 0 || p > 0) ? 1u : 0u;  // first write of level p + q
                        asm volatile(
                            "{\n\t.reg .pred pa;\n\t"
                            "setp.ne.b32 pa, %4, 0;\n\t"
                            "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, {%5, %5, %5, %5}, pa;\n\t}"
                            :: "r"(d), "l"(ad), "l"(bd), "r"(kTcIdesc), "r"(acc), "r"(0u) : "memory");
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
                const double w = scalbn(1.0, -8 * L - 12);                         // 2^-(8L+12)
#pragma unroll
                for (int c = 0; c < 16; ++c) s[c] = __fma_rn((double)(int)v[c], w, s[c]);   // exact products
            }
            if (rv) {
#pragma unroll
                for (int c = 0; c < 16; ++c) {
                    const int i = nt * kTcN + cb * 16 + c;
                    if (i < a.n_f) P[i] = scalbn(s[c], t.eU + 1);
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" :: "r"(tmem) : "memory");
}

}  // namespace syn
