// k_ozaki.cu -- K4/K5: an FP64 DGEMM task variant on the INT8 tensor cores
// (Ozaki scheme I), SURVEY.md SS8(f) NEXT-1.
//
// The paper's task model keeps one task interface with several implementation
// variants, chosen from the platform description (task
// repository and static pre-selection L1307-1326).  This file is the second
// variant of the DGEMM task (the first is K1, FP64 DMMA); the runtime picks it
// when the Worker's PDL property DGEMM_VARIANT is "ozaki" (K4).
//
// Method (error-free splitting into integer slices; Ozaki, Ogita, Oishi,
// Rump 2012; here with 7-bit signed slices and exact INT32 accumulation):
//   row scale   a_ik = 2^{e_i} a'_ik, |a'_ik| < 1      (e_i from frexp(max_k |a_ik|))
//   col scale   b_kj = 2^{f_j} b'_kj, |b'_kj| < 1
//   slices      a' = sum_{s<S} 2^{-7(s+1)} A_s,  A_s in [-127,127]  (truncation; exact FP64 ops)
//   product     C_ij ~= 2^{e_i+f_j} sum_{d<S} 2^{-7(d+2)} [ sum_{s+t=d} A_s B_t ]_ij
// Each diagonal d is ONE int8 GEMM with K' = (d+1) K: the slices are stored
// concatenated along K ([A_0|A_1|...] and, for B^T, in reverse order
// [...|B_1|B_0]), so [A_0..A_d] . [B_d..B_0]^T is a contiguous K' window of
// both.  |sum| <= (d+1) K 127^2 < 2^31 for K chunks <= 16384 (S <= 8), so the
// INT32 TMEM accumulation is exact; the epilogue scales by the exact power of
// two and accumulates the S diagonals into the FP64 C (smallest first).
// Representation error: |a - sum| < 2^{e_i - 7S}; with S = 7 the scaled error
// versus D = |A||B| is <= ~2^-45 for data whose rows / columns do not span a
// wide dynamic range (R19).  Inputs must be finite.
//
// GEMM kernel: the K2 v3 CTA-pair structure with tcgen05.mma.cta_group::2
// .kind::i8 (M = 256, N = 256, K = 32 per instruction), 6-stage TMA ring of
// 128-byte K blocks, INT32 accumulator in TMEM (256 columns), 16 epilogue
// warps converting TMEM -> FP64 and read-modify-writing C.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <algorithm>

#include "kernels.h"
#include "ptx.cuh"
#include "tcgen05.cuh"

namespace pdlk {

// ------------------------------------------------------------------------
// K5: slicing pre-pass
// ------------------------------------------------------------------------

// Scale exponent of a row / column from its non-negative finite max:
// max < 2^e (0 -> 0).  Round-to-nearest slicing (rn) additionally needs
// 128 * max * 2^-e < 127.5 so the first rint() stays within [-127, 127].
__device__ __forceinline__ int exp_of_max(double mx, int rn) {
    if (!(mx > 0.0)) return 0;
    int e;
    const double m = frexp(mx, &e);
    if (rn && m * 128.0 >= 127.5) ++e;
    return e;
}

// x 2^E (as ldexp): one DMUL by the bit-built power of two in the normal range
__device__ __forceinline__ double ldexp_fast(double x, int E) {
    if (E >= -1022 && E <= 1023) return x * __longlong_as_double((long long)(1023 + E) << 52);
    return ldexp(x, E);
}

// One slicing step: v <- 128 v, q = round(v) (trunc or nearest), v <- v - q
// (all exact in FP64).  trunc: |q| <= 127, remainders in (-1,1); nearest:
// |q| <= 127 for the first slice, <= 64 after, remainders in [-1/2, 1/2].
// Returns q as an int.  Nearest rounding runs on the FP64 pipe only: t =
// fma(v, 128, 1.5 * 2^52) = magic + rint(128 v) (|128 v| < 2^51), q = t - magic,
// v = fma(v, 128, -q) (exact), and q's low word is the int -- no FRND / F2I on the
// quarter-rate conversion unit.
__device__ __forceinline__ int slice_q(double &v, int rn) {
    if (rn) {
        const double magic = 6755399441055744.0;
        const double t = fma(v, 128.0, magic);
        const double q = t - magic;
        v = fma(v, 128.0, -q);
        return __double2loint(t);
    }
    v *= 128.0;
    const double q = trunc(v);
    v -= q;
    return (int)q;
}

// One CTA per row (grid-stride): A (M x K, lda) -> A8 rows [c][s][kk].
// T = double (FP64 task) or float (FP32 task; promoted exactly to double).
template <typename T>
__global__ void oz_split_rows_kernel(const T *__restrict__ A, int64_t lda, int64_t M, int64_t K, int S,
                                     int64_t Kc, int nch, int8_t *__restrict__ A8, int64_t ld8,
                                     int *__restrict__ ea, int rn) {
    __shared__ double red[32];
    const int64_t Kpad = (int64_t)nch * Kc;
    for (int64_t i = blockIdx.x; i < M; i += gridDim.x) {
        const T *row = A + i * lda;
        double mx = 0.0;
        for (int64_t k = threadIdx.x; k < K; k += blockDim.x) mx = fmax(mx, fabs((double)row[k]));
        for (int o = 16; o; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = mx;
        __syncthreads();
        if (threadIdx.x < 32) {
            mx = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : 0.0;
            for (int o = 16; o; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
            if (threadIdx.x == 0) red[0] = mx;
        }
        __syncthreads();
        const int e = exp_of_max(red[0], rn);
        if (threadIdx.x == 0) ea[i] = e;
        int8_t *out = A8 + i * ld8;
        // groups of 8 consecutive k (Kc % 128 == 0: a group never straddles a chunk);
        // one 8-byte store per slice per group
        for (int64_t k8 = (int64_t)threadIdx.x * 8; k8 < Kpad; k8 += (int64_t)blockDim.x * 8) {
            double v[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = (k8 + j < K) ? ldexp_fast((double)row[k8 + j], -e) : 0.0;
            const int64_t c = k8 / Kc, kk = k8 - c * Kc;
            int8_t *o = out + (c * S) * Kc + kk;
            for (int s = 0; s < S; ++s) {
                uint64_t pk = 0;
#pragma unroll
                for (int j = 0; j < 8; ++j) pk |= (uint64_t)(uint8_t)slice_q(v[j], rn) << (8 * j);
                *reinterpret_cast<uint64_t *>(o + (int64_t)s * Kc) = pk;
            }
        }
        __syncthreads();
    }
}

// Column max |b| of B (K x N): bits of the non-negative max via atomicMax.
template <typename T>
__global__ void oz_colmax_kernel(const T *__restrict__ B, int64_t ldb, int64_t K, int64_t N,
                                 unsigned long long *__restrict__ bmax) {
    const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (n >= N) return;
    const int64_t k0 = (int64_t)blockIdx.y * 256, k1 = min(K, k0 + 256);
    double mx = 0.0;
    for (int64_t k = k0; k < k1; ++k) mx = fmax(mx, fabs((double)B[k * ldb + n]));
    atomicMax(bmax + n, (unsigned long long)__double_as_longlong(mx));
}

// B (K x N) -> Bt8 (N rows of [c][S-1-s][kk]) through a shared tile stored
// transposed (32 n rows x KT k, pitch KT + 2 doubles): coalesced loads along n,
// then each thread slices KG groups of 8 consecutive k of one column, read as
// 16-byte shared loads (conflict-free per quarter-warp) -> one 8-byte store per
// slice and group.  KT = 64 for FP64 inputs, 128 for FP32 (twice the work per CTA
// for the half-size elements).
template <typename T>
__global__ void __launch_bounds__(256) oz_split_cols_t_kernel(
    const T *__restrict__ B, int64_t ldb, int64_t K, int64_t N, int S, int64_t Kc, int nch,
    const unsigned long long *__restrict__ bmax, int8_t *__restrict__ Bt8, int64_t ld8, int *__restrict__ fb,
    int rn) {
    constexpr int KG = sizeof(T) == 4 ? 2 : 1, KT = 64 * KG, PITCH = KT + 2;
    __shared__ __align__(16) double t[32 * PITCH];
    const int64_t k0 = (int64_t)blockIdx.y * KT, n0 = (int64_t)blockIdx.x * 32;
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;   // 32 x 8
#pragma unroll
    for (int r = ty; r < KT; r += 8) {
        const int64_t k = k0 + r, n = n0 + tx;
        t[tx * PITCH + r] = (k < K && n < N) ? (double)B[k * ldb + n] : 0.0;
    }
    __syncthreads();
    const int64_t Kpad = (int64_t)nch * Kc;
    const int nl = threadIdx.x >> 3, g = threadIdx.x & 7;    // column, group of 8 k
    const int64_t n = n0 + nl;
    if (n >= N) return;
    const int f = exp_of_max(__longlong_as_double((long long)bmax[n]), rn);
    if (blockIdx.y == 0 && g == 0) fb[n] = f;
#pragma unroll
    for (int u = 0; u < KG; ++u) {
        const int gl = g + 8 * u;                            // group within the tile
        const int64_t k8 = k0 + 8 * gl;
        if (k8 >= Kpad) break;
        double v[8];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const double2 x = *reinterpret_cast<const double2 *>(&t[nl * PITCH + 8 * gl + 2 * j]);
            v[2 * j] = ldexp_fast(x.x, -f);
            v[2 * j + 1] = ldexp_fast(x.y, -f);
        }
        const int64_t c = k8 / Kc, kk = k8 - c * Kc;
        int8_t *o = Bt8 + n * ld8 + (c * S) * Kc + kk;
        for (int s = 0; s < S; ++s) {
            uint64_t pk = 0;
#pragma unroll
            for (int j = 0; j < 8; ++j) pk |= (uint64_t)(uint8_t)slice_q(v[j], rn) << (8 * j);
            *reinterpret_cast<uint64_t *>(o + (int64_t)(S - 1 - s) * Kc) = pk;
        }
    }
}

// ------------------------------------------------------------------------
// K4: int8 CTA-pair GEMM of one diagonal, FP64 epilogue
// ------------------------------------------------------------------------
namespace koz {
// NSUB N=256 sub-tiles per cluster: NSUB = 2 gives 256 x 512 cluster tiles
// (two MMAs per K step into TMEM columns [0,256) and [256,512)), halving the
// A-panel traffic per output element; NSUB = 1 for narrow problems.
constexpr int BM = 128, BN1 = 256, BNH = 128;
constexpr int BK = 128, UMMA_K = 32;
constexpr int A_BYTES = BM * BK;        // 16 KiB
constexpr int B_BYTES = BNH * BK;       // 16 KiB per N=256 sub-tile
constexpr int FIRST_EPI_WARP = 2;
// Raster group (cluster-tile rows sweeping the columns together) from the K extent
// of the launch: the group's A strips (256 rows x K' bytes each) should stay in L2
// while the columns go by, so long diagonals take small groups.  Sweeps at C4
// (profiles/r01_sweep_group*.txt): K' = 16384 -> 16 (Ozaki-II: DRAM 5.37 -> 3.52
// GB per launch, 182.8 -> 189.7 TFLOP/s; 32, 64 thrash), FP32 Ozaki (K' <= 3K) 8
// over 4, FP64 Ozaki-I (K' <= 6K) 4 ~ 8.  PDL_GROUP_M overrides.
inline int group_for_k(int64_t kd) {
    const int64_t strip = 256 * kd;
    int g = 16;
    while (g > 4 && (int64_t)g * strip > ((int64_t)96 << 20)) g >>= 1;
    return raster_group_m(g);
}
// OCC = CTAs per SM.  OCC = 1: one CTA (pair) owns the SM pair, 16 epilogue
// warps, a 6-stage ring (4 for NSUB = 2).  OCC = 2 (NSUB = 1 only): two CTA pairs
// share each SM pair, each with 256 TMEM columns, a 3-stage ring and 8 epilogue
// warps, so one pair's epilogue (and prologue) overlaps the other's mainloop.
template <int NSUB, int OCC = 1> struct Cfg {
    static_assert(OCC == 1 || NSUB == 1, "two CTAs per SM need the 256-column tile");
    static constexpr int BN = BN1 * NSUB;
    static constexpr int STAGE_BYTES = A_BYTES + NSUB * B_BYTES;
    static constexpr int STAGES = OCC == 2 ? 3 : (6 * (A_BYTES + B_BYTES)) / STAGE_BYTES;   // 6, 4 or 3
    static constexpr int EPI_WARPS = OCC == 2 ? 8 : 16;
    static constexpr int THREADS = (FIRST_EPI_WARP + EPI_WARPS) * 32;
    static constexpr int EPI_COLS = 256 * NSUB / (EPI_WARPS / 4);
    static constexpr int TMEM_COLS = 256 * NSUB;
    static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 + 256;
};
}  // namespace koz

__host__ __device__ constexpr uint32_t idesc_i8(int M, int N) {
    return (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// x * 2^E for an int32 x, correctly rounded (as ldexp): one DMUL by the power
// of two built from its bits when 2^E is a normal double; otherwise an exact
// first step to the edge of the normal range, then one rounding multiply.
__device__ __forceinline__ double pow2_normal(int E) {   // E in [-1022, 1023]
    return __longlong_as_double((long long)(1023 + E) << 52);
}
// int32 -> double exactly on the FP64 pipe (the conversion unit runs at a quarter
// of its rate): the bits 0x43380000:(x ^ 2^31) are 1.5 * 2^52 + 2^31 + x.
__device__ __forceinline__ double i2d_exact(int32_t x) {
    return __hiloint2double(0x43380000, x ^ (int)0x80000000) - 6755401588539392.0;
}
__device__ __forceinline__ double scale_pow2(int32_t x, int E) {
    if (E >= -1022 && E <= 1023) return i2d_exact(x) * pow2_normal(E);
    const int E1 = E < 0 ? -1022 : 1023;
    const int E2 = max(-1022, min(1023, E - E1));
    return (i2d_exact(x) * pow2_normal(E1)) * pow2_normal(E2);
}

__device__ __forceinline__ void umma_i8_2sm(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                            uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}

template <int NSUB, typename TC, int OCC = 1>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(koz::Cfg<NSUB, OCC>::THREADS, OCC)
    oz_gemm_2sm_kernel(const __grid_constant__ CUtensorMap tA, const __grid_constant__ CUtensorMap tB,
                       TC *__restrict__ C, int64_t ldc, int M, int N, int Kd, const int *__restrict__ ea,
                       const int *__restrict__ fb, int scale_exp, int accumulate, int tiles_m, int tiles_n,
                       int group_m, int vec_ok, int modulus, unsigned mod_magic) {
    using namespace koz;
    using CF = Cfg<NSUB, OCC>;
    constexpr int BN = CF::BN, STAGES = CF::STAGES, STAGE_BYTES = CF::STAGE_BYTES;
    constexpr int EPI_COLS = CF::EPI_COLS, TMEM_COLS = CF::TMEM_COLS;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t base = (smem_u32(smem_raw) + 1023u) & ~1023u;
    const uint32_t bar_full = base + STAGES * STAGE_BYTES;
    const uint32_t bar_empty = bar_full + STAGES * 8;
    const uint32_t bar_tfull = bar_empty + STAGES * 8;
    const uint32_t tmem_slot = bar_tfull + 8;
    uint8_t *const gbase = smem_raw + (base - smem_u32(smem_raw));
    volatile uint32_t *tmem_slot_ptr = reinterpret_cast<volatile uint32_t *>(gbase + (tmem_slot - base));

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = cluster_ctarank();
    int tm, tn;
    raster_tile(blockIdx.x >> 1, tiles_m, tiles_n, group_m, &tm, &tn);
    const int m0 = tm * (2 * BM) + (int)rank * BM;
    const int nb0 = tn * BN + (int)rank * BNH;   // + j * 256 for sub-tile j

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(bar_full + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, 1);
        }
        mbar_init(bar_tfull, 1);
        fence_barrier_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(tmem_slot),
                     "n"(TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync_all();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem_base = *tmem_slot_ptr;
    const int nk = Kd / BK;

    if (warp == 0) {
        if (lane == 0) {
            tma_prefetch_desc(&tA);
            tma_prefetch_desc(&tB);
            for (int kb = 0; kb < nk; ++kb) {
                const int s = kb % STAGES;
                const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
                mbar_wait(bar_empty + 8 * s, ph ^ 1u);
                const uint32_t fb_leader = mapa_shared(bar_full + 8 * s, 0);
                if (rank == 0) mbar_arrive_expect_tx(bar_full + 8 * s, 2 * STAGE_BYTES);
                const uint32_t st = base + s * STAGE_BYTES;
                tma_load_2d_2sm(st, &tA, fb_leader, kb * BK, m0);
#pragma unroll
                for (int j = 0; j < NSUB; ++j)
                    tma_load_2d_2sm(st + A_BYTES + j * B_BYTES, &tB, fb_leader, kb * BK, nb0 + j * BN1);
            }
        }
    } else if (warp == 1) {
        if (rank == 0 && lane == 0) {
            constexpr uint32_t idesc = idesc_i8(2 * BM, BN1);
            for (int kb = 0; kb < nk; ++kb) {
                const int s = kb % STAGES;
                const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
                mbar_wait(bar_full + 8 * s, ph);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const uint32_t st = base + s * STAGE_BYTES;
#pragma unroll
                for (int kk = 0; kk < BK / UMMA_K; ++kk) {
                    const uint32_t off = kk * UMMA_K;   // 32 bytes of K per instruction
#pragma unroll
                    for (int j = 0; j < NSUB; ++j)
                        umma_i8_2sm(tmem_base + j * BN1, umma_desc_k_sw128(st + off),
                                    umma_desc_k_sw128(st + A_BYTES + j * B_BYTES + off), idesc, (kb | kk) ? 1u : 0u);
                }
                umma_commit_2sm(bar_empty + 8 * s);
            }
            umma_commit_2sm(bar_tfull);
        }
        __syncwarp();
    } else {
        const int e = warp - FIRST_EPI_WARP;
        const int q = warp & 3;
        const int cg = e >> 2;
        const uint32_t tl = tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(cg * EPI_COLS);
        mbar_wait(bar_tfull, 0);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if constexpr (sizeof(TC) == 1) {
            // Ozaki-II (K6): the exact INT32 sum reduced mod m into a byte plane
            // (C = plane, ldc = its row pitch, 16-byte aligned).  Each thread owns
            // its TMEM lane = row and stores 16 consecutive residues per step.
            // |x| <= Kc 2^14 <= 2^30, so xb = x + bias (bias = m ceil(2^30 / m)) lies in
            // [0, 2^31 + m) and xb mod m = xb - m umulhi(xb, mag) >> 7 exactly, with
            // mag = ceil(2^39 / m) < 2^32 (e = mag m - 2^39 < m and xb e < 2^39):
            // four integer operations, no conversions.
            const int row = tm * (2 * BM) + (int)rank * BM + q * 32 + lane;
            const int cbase = tn * BN + cg * EPI_COLS;
            uint8_t *prow = reinterpret_cast<uint8_t *>(C) + (int64_t)row * ldc + cbase;
            const uint32_t mm = (uint32_t)modulus, bias = mm * ((1u << 30) / mm + 1u);
#pragma unroll 1
            for (int c0 = 0; c0 < EPI_COLS; c0 += 16) {
                uint32_t r[16];
                tmem_ld16(tl + c0, r);
                if (row >= M) continue;
                uint32_t pk[4];
#pragma unroll
                for (int w4 = 0; w4 < 4; ++w4) {
                    uint32_t res[4];
#pragma unroll
                    for (int b = 0; b < 4; ++b) {
                        const uint32_t xb = r[4 * w4 + b] + bias;
                        res[b] = xb - (__umulhi(xb, mod_magic) >> 7) * mm;
                    }
                    pk[w4] = __byte_perm(__byte_perm(res[0], res[1], 0x0040), __byte_perm(res[2], res[3], 0x0040), 0x5410);
                }
                if (cbase + c0 + 16 <= N) {
                    *reinterpret_cast<uint4 *>(prow + c0) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                } else {
#pragma unroll
                    for (int jj = 0; jj < 16; ++jj)
                        if (cbase + c0 + jj < N) prow[c0 + jj] = (uint8_t)(pk[jj >> 2] >> (8 * (jj & 3)));
                }
            }
        } else {
        // TMEM lane = C row: each thread converts its own row (exact power-of-two
        // scaling), then the warp transposes 32 rows x 16 columns through shared
        // memory (the operand ring is idle once bar_tfull fired) so that the C
        // read-modify-write is row-contiguous: 8 lanes x 16 B per row, 4 rows per
        // instruction.  128B XOR swizzle: both phases are bank-conflict free.
        const int row0 = tm * (2 * BM) + (int)rank * BM + q * 32;   // first row of this warp
        const int row = row0 + lane;
        const int cbase = tn * BN + cg * EPI_COLS;
        const int er = row < M ? ea[row] + scale_exp : 0;
        const uint32_t stg = base + (uint32_t)e * 4096u;               // 32 x 128 B per warp
        const int rsub = lane >> 3, kch = lane & 7;                    // read phase: row in 4, 16 B chunk
        const bool vec = vec_ok != 0;
#pragma unroll 1
        for (int c0 = 0; c0 < EPI_COLS; c0 += 16) {
            uint32_t r[16];
            tmem_ld16(tl + c0, r);
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                double v0 = 0.0, v1 = 0.0;
                if (row < M) {
                    const int col = cbase + c0 + 2 * k;
                    v0 = scale_pow2((int32_t)r[2 * k], er + (col < N ? fb[col] : 0));   // exact
                    v1 = scale_pow2((int32_t)r[2 * k + 1], er + (col + 1 < N ? fb[col + 1] : 0));
                }
                const uint32_t a = stg + (uint32_t)lane * 128u + (((uint32_t)k ^ ((uint32_t)lane & 7u)) << 4);
                asm volatile("st.shared.v2.f64 [%0], {%1, %2};" ::"r"(a), "d"(v0), "d"(v1) : "memory");
            }
            __syncwarp();
            // the C loads of four rows are issued before their stores (two DRAM
            // round trips per 32 x 16 chunk instead of eight dependent ones)
            const int col = cbase + c0 + 2 * kch;
            const bool vcol = vec && col + 1 < N;
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                double2 val[4], old[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int rr = 4 * (4 * h + u) + rsub;             // row within the warp's 32
                    const uint32_t a = stg + (uint32_t)rr * 128u + (((uint32_t)kch ^ ((uint32_t)rr & 7u)) << 4);
                    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(val[u].x), "=d"(val[u].y) : "r"(a) : "memory");
                    old[u] = make_double2(0.0, 0.0);
                    const int grow = row0 + rr;
                    if (accumulate && vcol && grow < M) {
                        const TC *cp = C + (int64_t)grow * ldc + col;
                        if constexpr (sizeof(TC) == 8) {
                            old[u] = __ldcs(reinterpret_cast<const double2 *>(cp));
                        } else {
                            const float2 o = __ldcs(reinterpret_cast<const float2 *>(cp));
                            old[u] = make_double2((double)o.x, (double)o.y);
                        }
                    }
                }
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int grow = row0 + 4 * (4 * h + u) + rsub;
                    if (grow >= M) continue;
                    TC *cp = C + (int64_t)grow * ldc + col;
                    const double v0 = val[u].x, v1 = val[u].y;
                    if (vcol) {
                        // streaming (evict-first) C traffic keeps the slice panels in L2;
                        // FP32 task: each diagonal adds in double and rounds once to float
                        if constexpr (sizeof(TC) == 8)
                            __stcs(reinterpret_cast<double2 *>(cp), make_double2(old[u].x + v0, old[u].y + v1));
                        else
                            __stcs(reinterpret_cast<float2 *>(cp),
                                   make_float2((float)(old[u].x + v0), (float)(old[u].y + v1)));
                    } else {
                        if (col < N) cp[0] = (TC)((accumulate ? (double)cp[0] : 0.0) + v0);
                        if (col + 1 < N) cp[1] = (TC)((accumulate ? (double)cp[1] : 0.0) + v1);
                    }
                }
            }
            __syncwarp();
        }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync_all();
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(TMEM_COLS));
    }
}

// K6, persistent: one CTA pair per TPC walks the work items (modulus t, cluster
// tile) of all nmod residue GEMMs of a K chunk, modulus-major (item = cluster,
// cluster + clusters, ...), so the last partial round of tiles is paid once per
// K chunk instead of once per modulus.  The operands of modulus t are the K
// columns [t Kd, (t+1) Kd) of the tensor maps (the residues of a row are
// contiguous per modulus), its residues go to plane t of R.  Barriers and TMEM
// are set up once; the producer runs ahead into the next item while the
// epilogue drains the accumulator, and the MMA warp starts the next item as soon
// as both CTAs' epilogue warps have read TMEM (bar_tempty on the leader, 2 x
// EPI_WARPS arrivals), so only the TMEM read -- not the prologue, pipeline fill,
// residue arithmetic and stores -- sits between two items' MMAs.  Epilogue as
// oz_gemm_2sm_kernel<NSUB, uint8_t>.
struct Oz2Moduli {
    int m[OZ2_MAX_MODULI];
    unsigned magic[OZ2_MAX_MODULI];   // ceil(2^39 / m): exact division-by-constant multiplier
};

template <int NSUB>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(koz::Cfg<NSUB, 1>::THREADS, 1)
    oz2_gemm_persistent_kernel(const __grid_constant__ CUtensorMap tA, const __grid_constant__ CUtensorMap tB,
                               uint8_t *__restrict__ R, int64_t ldr, int64_t plane, int M, int N, int Kd,
                               int tiles_m, int tiles_n, int group_m, int nmod, const __grid_constant__ Oz2Moduli mods,
                               int hints) {
    using namespace koz;
    using CF = Cfg<NSUB, 1>;
    constexpr int BN = CF::BN, STAGES = CF::STAGES, STAGE_BYTES = CF::STAGE_BYTES;
    constexpr int EPI_COLS = CF::EPI_COLS, TMEM_COLS = CF::TMEM_COLS, EPI_WARPS = CF::EPI_WARPS;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t base = (smem_u32(smem_raw) + 1023u) & ~1023u;
    const uint32_t bar_full = base + STAGES * STAGE_BYTES;
    const uint32_t bar_empty = bar_full + STAGES * 8;
    const uint32_t bar_tfull = bar_empty + STAGES * 8;
    const uint32_t bar_tempty = bar_tfull + 8;
    const uint32_t tmem_slot = bar_tempty + 8;
    uint8_t *const gbase = smem_raw + (base - smem_u32(smem_raw));
    volatile uint32_t *tmem_slot_ptr = reinterpret_cast<volatile uint32_t *>(gbase + (tmem_slot - base));

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = cluster_ctarank();
    const int ntiles = tiles_m * tiles_n, nclusters = (int)(gridDim.x >> 1), cl = (int)(blockIdx.x >> 1);
    const int nitems = nmod * ntiles;

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(bar_full + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, 1);
        }
        mbar_init(bar_tfull, 1);
        mbar_init(bar_tempty, 2 * EPI_WARPS);
        fence_barrier_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(tmem_slot),
                     "n"(TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync_all();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem_base = *tmem_slot_ptr;
    const int nk = Kd / BK;

    if (warp == 0) {
        if (lane == 0) {
            tma_prefetch_desc(&tA);
            tma_prefetch_desc(&tB);
            // hints & 1: A strips (reused across the raster group's column sweep) evict_last,
            // B strips (read by one wave of the group) evict_first
            const uint64_t pol_a = l2_policy_evict_last(), pol_b = l2_policy_evict_first();
            uint32_t it = 0;
            for (int item = cl; item < nitems; item += nclusters) {
                const int t = item / ntiles, tile = item - t * ntiles;
                int tm, tn;
                raster_tile(tile, tiles_m, tiles_n, group_m, &tm, &tn);
                const int m0 = tm * (2 * BM) + (int)rank * BM;
                const int nb0 = tn * BN + (int)rank * BNH;
                // hints & 4: odd rounds of tiles walk K backwards, so a round starts on the
                // K blocks of the (shared) A strips the previous round touched last and
                // still finds them in L2 (integer sums: the order does not change a bit)
                const bool rev = (hints & 4) && (((item / nclusters) & 1) != 0);
                for (int kb = 0; kb < nk; ++kb, ++it) {
                    const uint32_t s = it % STAGES, ph = (it / STAGES) & 1u;
                    mbar_wait(bar_empty + 8 * s, ph ^ 1u);
                    const uint32_t fb_leader = mapa_shared(bar_full + 8 * s, 0);
                    if (rank == 0) mbar_arrive_expect_tx(bar_full + 8 * s, 2 * STAGE_BYTES);
                    const uint32_t st = base + s * STAGE_BYTES;
                    const int kx = t * Kd + (rev ? nk - 1 - kb : kb) * BK;
                    if (hints & 1) {
                        tma_load_2d_2sm_hint(st, &tA, fb_leader, kx, m0, pol_a);
#pragma unroll
                        for (int j = 0; j < NSUB; ++j)
                            tma_load_2d_2sm_hint(st + A_BYTES + j * B_BYTES, &tB, fb_leader, kx, nb0 + j * BN1, pol_b);
                    } else {
                        tma_load_2d_2sm(st, &tA, fb_leader, kx, m0);
#pragma unroll
                        for (int j = 0; j < NSUB; ++j)
                            tma_load_2d_2sm(st + A_BYTES + j * B_BYTES, &tB, fb_leader, kx, nb0 + j * BN1);
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (rank == 0 && lane == 0) {
            constexpr uint32_t idesc = idesc_i8(2 * BM, BN1);
            uint32_t it = 0, ti = 0;
            for (int item = cl; item < nitems; item += nclusters, ++ti) {
                mbar_wait(bar_tempty, (ti & 1u) ^ 1u);   // both CTAs' epilogues have read TMEM
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                for (int kb = 0; kb < nk; ++kb, ++it) {
                    const uint32_t s = it % STAGES, ph = (it / STAGES) & 1u;
                    mbar_wait(bar_full + 8 * s, ph);
                    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                    const uint32_t st = base + s * STAGE_BYTES;
#pragma unroll
                    for (int kk = 0; kk < BK / UMMA_K; ++kk) {
                        const uint32_t off = kk * UMMA_K;
#pragma unroll
                        for (int j = 0; j < NSUB; ++j)
                            umma_i8_2sm(tmem_base + j * BN1, umma_desc_k_sw128(st + off),
                                        umma_desc_k_sw128(st + A_BYTES + j * B_BYTES + off), idesc,
                                        (kb | kk) ? 1u : 0u);
                    }
                    umma_commit_2sm(bar_empty + 8 * s);
                }
                umma_commit_2sm(bar_tfull);
            }
        }
        __syncwarp();
    } else {
        const int e = warp - FIRST_EPI_WARP;
        const int q = warp & 3;
        const int cg = e >> 2;
        const uint32_t tl = tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(cg * EPI_COLS);
        const uint32_t tempty_leader = mapa_shared(bar_tempty, 0);
        uint32_t ti = 0;
        for (int item = cl; item < nitems; item += nclusters, ++ti) {
            const int t = item / ntiles, tile = item - t * ntiles;
            const uint32_t mm = (uint32_t)mods.m[t], bias = mm * ((1u << 30) / mm + 1u);
            const unsigned mod_magic = mods.magic[t];
            int tm, tn;
            raster_tile(tile, tiles_m, tiles_n, group_m, &tm, &tn);
            const int row = tm * (2 * BM) + (int)rank * BM + q * 32 + lane;
            const int cbase = tn * BN + cg * EPI_COLS;
            uint8_t *prow = R + (int64_t)t * plane + (int64_t)row * ldr + cbase;
            mbar_wait(bar_tfull, ti & 1u);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll 1
            for (int c0 = 0; c0 < EPI_COLS; c0 += 16) {
                uint32_t r[16];
                tmem_ld16(tl + c0, r);
                if (c0 + 16 == EPI_COLS) {   // this warp's last TMEM read is complete
                    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
                    __syncwarp();
                    if (lane == 0) mbar_arrive_cluster(tempty_leader);
                }
                if (row >= M) continue;
                uint32_t pk[4];
#pragma unroll
                for (int w4 = 0; w4 < 4; ++w4) {
                    uint32_t res[4];
#pragma unroll
                    for (int b = 0; b < 4; ++b) {
                        const uint32_t xb = r[4 * w4 + b] + bias;
                        res[b] = xb - (__umulhi(xb, mod_magic) >> 7) * mm;
                    }
                    pk[w4] = __byte_perm(__byte_perm(res[0], res[1], 0x0040), __byte_perm(res[2], res[3], 0x0040), 0x5410);
                }
                if (cbase + c0 + 16 <= N) {
                    // hints & 2: streaming (evict-first) plane stores keep the operand strips in L2
                    if (hints & 2)
                        __stcs(reinterpret_cast<uint4 *>(prow + c0), make_uint4(pk[0], pk[1], pk[2], pk[3]));
                    else
                        *reinterpret_cast<uint4 *>(prow + c0) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                } else {
#pragma unroll
                    for (int jj = 0; jj < 16; ++jj)
                        if (cbase + c0 + jj < N) prow[c0 + jj] = (uint8_t)(pk[jj >> 2] >> (8 * (jj & 3)));
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync_all();
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(TMEM_COLS));
    }
}

// ------------------------------------------------------------------------
// host side
// ------------------------------------------------------------------------
OzakiLayout ozaki_layout(int64_t rows, int64_t cols, int64_t K, int S) {
    OzakiLayout L;
    L.S = S;
    L.nch = (int)((K + OZ_KC_MAX - 1) / OZ_KC_MAX);
    if (L.nch < 1) L.nch = 1;
    const int64_t per = (K + L.nch - 1) / L.nch;
    L.Kc = ((per + koz::BK - 1) / koz::BK) * koz::BK;
    L.ld8 = (int64_t)L.nch * S * L.Kc;
    L.a8_bytes = (size_t)rows * L.ld8;
    L.b8_bytes = (size_t)cols * L.ld8;
    return L;
}

static int split_ctas() {
    const char *e = getenv("PDL_SPLIT_CTAS");
    return e && atoi(e) > 0 ? atoi(e) : 148 * 8;
}

template <typename T>
static cudaError_t split_a_impl(const T *A, int64_t lda, int64_t rows, int64_t K, const OzakiLayout &L, int8_t *A8,
                                int *ea, cudaStream_t s) {
    if (rows <= 0) return cudaSuccess;
    int blocks = (int)(rows < split_ctas() ? rows : split_ctas());
    oz_split_rows_kernel<T><<<blocks, 256, 0, s>>>(A, lda, rows, K, L.S, L.Kc, L.nch, A8, L.ld8, ea, L.rn);
    return cudaGetLastError();
}

template <typename T>
static cudaError_t split_b_impl(const T *B, int64_t ldb, int64_t K, int64_t cols, const OzakiLayout &L, int8_t *Bt8,
                                int *fb, unsigned long long *bmax, cudaStream_t s) {
    if (cols <= 0) return cudaSuccess;
    cudaError_t e = cudaMemsetAsync(bmax, 0, (size_t)cols * sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    if (K > 0) {
        dim3 g1((unsigned)((cols + 255) / 256), (unsigned)((K + 255) / 256));
        oz_colmax_kernel<T><<<g1, 256, 0, s>>>(B, ldb, K, cols, bmax);
    }
    const int64_t Kpad = (int64_t)L.nch * L.Kc;
    const int64_t kt = sizeof(T) == 4 ? 128 : 64;   // k rows per CTA (oz_split_cols_t_kernel KT)
    dim3 g2((unsigned)((cols + 31) / 32), (unsigned)((Kpad + kt - 1) / kt));
    oz_split_cols_t_kernel<T><<<g2, 256, 0, s>>>(B, ldb, K, cols, L.S, L.Kc, L.nch, bmax, Bt8, L.ld8, fb, L.rn);
    return cudaGetLastError();
}

cudaError_t launch_ozaki_split_a(const double *A, int64_t lda, int64_t rows, int64_t K, const OzakiLayout &L,
                                 int8_t *A8, int *ea, cudaStream_t s) {
    return split_a_impl(A, lda, rows, K, L, A8, ea, s);
}
cudaError_t launch_ozaki_split_a(const float *A, int64_t lda, int64_t rows, int64_t K, const OzakiLayout &L,
                                 int8_t *A8, int *ea, cudaStream_t s) {
    return split_a_impl(A, lda, rows, K, L, A8, ea, s);
}
cudaError_t launch_ozaki_split_b(const double *B, int64_t ldb, int64_t K, int64_t cols, const OzakiLayout &L,
                                 int8_t *Bt8, int *fb, unsigned long long *bmax, cudaStream_t s) {
    return split_b_impl(B, ldb, K, cols, L, Bt8, fb, bmax, s);
}
cudaError_t launch_ozaki_split_b(const float *B, int64_t ldb, int64_t K, int64_t cols, const OzakiLayout &L,
                                 int8_t *Bt8, int *fb, unsigned long long *bmax, cudaStream_t s) {
    return split_b_impl(B, ldb, K, cols, L, Bt8, fb, bmax, s);
}

static bool map_i8(EncodeTiledFn enc, CUtensorMap *m, const int8_t *ptr, uint64_t kd, uint64_t rows, uint64_t ld,
                   uint32_t box_rows) {
    cuuint64_t dims[2] = {kd, rows};
    cuuint64_t strides[1] = {ld};
    cuuint32_t box[2] = {(cuuint32_t)koz::BK, box_rows};
    cuuint32_t es[2] = {1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<int8_t *>(ptr), dims, strides, box, es,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Kernel shape for one rectangle: 0 = 256 x 512 cluster tiles (NSUB 2), 1 = 256 x
// 256 (NSUB 1), 2 = 256 x 256 with two CTA pairs per SM pair (OCC 2).  Exact INT32
// sums: the shape does not change a bit of C.  Default: 256 x 512 when it still
// gives >= 2 waves of CTA pairs (148 clusters), else 256 x 256 for parallelism.
// PDL_OZ_SHAPE = 512 | 256 | 256x2 overrides (PDL_OZ_NSUB = 1 | 2 is the older knob).
static int oz_shape(int64_t rows, int64_t cols) {
    using namespace koz;
    const int64_t clusters512 = ((rows + 2 * BM - 1) / (2 * BM)) * ((cols + 511) / 512);
    int shape = (cols > 256 && clusters512 >= worker_sms()) ? 0 : 1;
    if (const char *e = getenv("PDL_OZ_NSUB")) shape = atoi(e) == 1 ? 1 : 0;
    if (const char *e = getenv("PDL_OZ_SHAPE")) {
        if (!strcmp(e, "512")) shape = 0;
        else if (!strcmp(e, "256")) shape = 1;
        else if (!strcmp(e, "256x2")) shape = 2;
    }
    return shape;
}

template <typename TC>
static cudaError_t oz_set_attrs() {
    using namespace koz;
    int dev = 0;
    cudaGetDevice(&dev);
    static bool attr_done[64] = {false};
    if (dev < 64 && attr_done[dev]) return cudaSuccess;
    cudaError_t e = cudaFuncSetAttribute(oz_gemm_2sm_kernel<1, TC, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         Cfg<1, 1>::SMEM_BYTES);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(oz_gemm_2sm_kernel<2, TC, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 Cfg<2, 1>::SMEM_BYTES);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(oz_gemm_2sm_kernel<1, TC, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 Cfg<1, 2>::SMEM_BYTES);
    if (e != cudaSuccess) return e;
    if (dev < 64) attr_done[dev] = true;
    return cudaSuccess;
}

// Co-resident CTA pairs of the persistent K6 kernel (cudaOccupancyMaxActiveClusters,
// cached per device); sets its shared-memory attribute on first use.
static cudaError_t oz2_persistent_clusters(int *out) {
    using namespace koz;
    using CF = Cfg<2, 1>;
    int dev = 0;
    cudaGetDevice(&dev);
    static int cached[64] = {0};
    if (dev < 64 && cached[dev] > 0) {
        *out = cached[dev];
        return cudaSuccess;
    }
    cudaError_t e = cudaFuncSetAttribute(oz2_gemm_persistent_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         CF::SMEM_BYTES);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2 * 148, 1, 1);
    cfg.blockDim = dim3(CF::THREADS, 1, 1);
    cfg.dynamicSmemBytes = CF::SMEM_BYTES;
    cudaLaunchAttribute attr;
    attr.id = cudaLaunchAttributeClusterDimension;
    attr.val.clusterDim.x = 2;
    attr.val.clusterDim.y = 1;
    attr.val.clusterDim.z = 1;
    cfg.attrs = &attr;
    cfg.numAttrs = 1;
    int n = 0;
    e = cudaOccupancyMaxActiveClusters(&n, oz2_gemm_persistent_kernel<2>, &cfg);
    if (e != cudaSuccess) return e;
    if (n < 1) return cudaErrorInvalidConfiguration;
    if (dev < 64) cached[dev] = n;
    *out = n;
    return cudaSuccess;
}

// Co-resident CTA pairs for the launching Worker: an SM-partition Worker holds one
// pair per two of its SMs at most.
static cudaError_t oz2_worker_clusters(int *out) {
    cudaError_t e = oz2_persistent_clusters(out);
    if (e != cudaSuccess) return e;
    *out = std::max(1, std::min(*out, worker_sms() / 2));
    return cudaSuccess;
}

template <int NSUB, int OCC, typename TC>
static void oz_launch_one(const CUtensorMap &ta, const CUtensorMap &tb, TC *C, int64_t ldc, int64_t rows,
                          int64_t cols, int64_t kd, const int *ea, const int *fb, int scale_exp, int accumulate,
                          int vec_ok, int modulus, unsigned mod_magic, cudaStream_t stream) {
    using namespace koz;
    using CF = Cfg<NSUB, OCC>;
    const int tiles_m = (int)((rows + 2 * BM - 1) / (2 * BM)), tiles_n = (int)((cols + CF::BN - 1) / CF::BN);
    oz_gemm_2sm_kernel<NSUB, TC, OCC><<<2 * tiles_m * tiles_n, CF::THREADS, CF::SMEM_BYTES, stream>>>(
        ta, tb, C, ldc, (int)rows, (int)cols, (int)kd, ea, fb, scale_exp, accumulate, tiles_m, tiles_n,
        group_for_k(kd), vec_ok, modulus, mod_magic);
}

template <typename TC>
static void oz_launch(int shape, const CUtensorMap &ta, const CUtensorMap &tb, TC *C, int64_t ldc, int64_t rows,
                      int64_t cols, int64_t kd, const int *ea, const int *fb, int scale_exp, int accumulate,
                      int vec_ok, int modulus, unsigned mod_magic, cudaStream_t stream) {
    if (shape == 0)
        oz_launch_one<2, 1>(ta, tb, C, ldc, rows, cols, kd, ea, fb, scale_exp, accumulate, vec_ok, modulus, mod_magic,
                            stream);
    else if (shape == 1)
        oz_launch_one<1, 1>(ta, tb, C, ldc, rows, cols, kd, ea, fb, scale_exp, accumulate, vec_ok, modulus, mod_magic,
                            stream);
    else
        oz_launch_one<1, 2>(ta, tb, C, ldc, rows, cols, kd, ea, fb, scale_exp, accumulate, vec_ok, modulus, mod_magic,
                            stream);
}

// All diagonals and K chunks of one rectangle: S * nch int8 GEMM launches,
// smallest diagonal first; the first launch overwrites C.
template <typename TC>
static cudaError_t gemm_impl(EncodeTiledFn enc, const int8_t *A8, const int8_t *Bt8, const int *ea, const int *fb,
                             const OzakiLayout &L, TC *C, int64_t ldc, int64_t rows, int64_t cols, cudaStream_t stream,
                             int *launches) {
    using namespace koz;
    if (rows <= 0 || cols <= 0) return cudaSuccess;
    cudaError_t e0 = oz_set_attrs<TC>();
    if (e0 != cudaSuccess) return e0;
    const int shape = oz_shape(rows, cols);
    const int vec_ok = ((reinterpret_cast<uintptr_t>(C) & 15u) == 0 && ((ldc * sizeof(TC)) & 15) == 0) ? 1 : 0;
    int first = 1;
    for (int c = 0; c < L.nch; ++c) {
        for (int d = L.S - 1; d >= 0; --d) {
            const int64_t kd = (int64_t)(d + 1) * L.Kc;
            const int8_t *a = A8 + (int64_t)c * L.S * L.Kc;
            const int8_t *b = Bt8 + ((int64_t)c * L.S + (L.S - 1 - d)) * L.Kc;
            CUtensorMap ta, tb;
            if (!map_i8(enc, &ta, a, (uint64_t)kd, (uint64_t)rows, (uint64_t)L.ld8, BM) ||
                !map_i8(enc, &tb, b, (uint64_t)kd, (uint64_t)cols, (uint64_t)L.ld8, BNH))
                return cudaErrorInvalidValue;
            oz_launch<TC>(shape, ta, tb, C, ldc, rows, cols, kd, ea, fb, -7 * (d + 2), first ? 0 : 1, vec_ok, 0, 0u,
                          stream);
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return e;
            first = 0;
            if (launches) ++*launches;
        }
    }
    return cudaSuccess;
}

cudaError_t launch_ozaki_gemm(EncodeTiledFn enc, const int8_t *A8, const int8_t *Bt8, const int *ea, const int *fb,
                              const OzakiLayout &L, double *C, int64_t ldc, int64_t rows, int64_t cols,
                              cudaStream_t stream, int *launches) {
    return gemm_impl(enc, A8, Bt8, ea, fb, L, C, ldc, rows, cols, stream, launches);
}
cudaError_t launch_ozaki_gemm(EncodeTiledFn enc, const int8_t *A8, const int8_t *Bt8, const int *ea, const int *fb,
                              const OzakiLayout &L, float *C, int64_t ldc, int64_t rows, int64_t cols,
                              cudaStream_t stream, int *launches) {
    return gemm_impl(enc, A8, Bt8, ea, fb, L, C, ldc, rows, cols, stream, launches);
}

// Moduli per persistent K6 launch (host arithmetic).  A launch walks the tiles of
// a group of moduli (modulus-major), so a small rectangle (a multi-GPU chunk: < 1
// round of tiles per modulus) pays the idle tail of a last round once per launch
// instead of once per modulus.  Long launches lose L2 locality: at C4 (28 rounds
// per modulus) one launch for all 13 moduli read 2x the DRAM bytes (L2 hit 73 ->
// 62 %: the clusters drift apart over 360 rounds and the live strips spread) and
// the power-capped clock fell 10 %.  So: the fewest launches nl with at most
// kOz2MaxRounds rounds each (a single modulus may exceed it) that minimise the
// idle rounds sum_l (ceil(r_l) - r_l),
// moduli spread evenly (launch l: moduli [l n / nl, (l+1) n / nl)).
int oz2_launches_per_chunk(int n, int64_t rows, int64_t cols, int clusters) {
    constexpr double kOz2MaxRounds = 24.0;
    if (n <= 1 || rows <= 0 || cols <= 0 || clusters <= 0) return std::max(1, n);
    const int64_t tiles = ((rows + 2 * koz::BM - 1) / (2 * koz::BM)) * ((cols + 511) / 512);
    const double rmod = (double)tiles / clusters;   // rounds per modulus
    int nl = n;
    double best = 1e30;
    for (int L = 1; L <= n; ++L) {
        const int gmax = (n + L - 1) / L;   // the largest group of an even spread
        if (gmax > 1 && gmax * rmod > kOz2MaxRounds + 1e-9) continue;
        double idle = 0.0;
        for (int l = 0; l < L; ++l) {
            const double r = rmod * ((l + 1) * n / L - l * n / L);
            idle += std::ceil(r - 1e-9) - r;
        }
        if (idle < best - 1e-6) {
            best = idle;
            nl = L;
        }
    }
    return nl;
}

// Ozaki-II (K6): one INT8 GEMM per modulus and K chunk, each writing its byte
// plane of residues (k_ozaki2.cu builds the operands and rebuilds C).
cudaError_t launch_ozaki2_gemm(EncodeTiledFn enc, const int8_t *A8, const int8_t *Bt8, const Ozaki2Plan &P,
                               uint8_t *R, int64_t ldr, int64_t plane, int64_t rows, int64_t cols, cudaStream_t stream,
                               int *launches) {
    using namespace koz;
    if (rows <= 0 || cols <= 0) return cudaSuccess;
    if ((reinterpret_cast<uintptr_t>(R) & 15u) || (ldr & 15) || (plane & 15)) return cudaErrorInvalidValue;
    cudaError_t e0 = oz_set_attrs<uint8_t>();
    if (e0 != cudaSuccess) return e0;
    // persistent 256 x 512 tiles by default, small grids included: the moduli of a
    // launch fill the rounds (PDL_OZ2_PERSIST=0: one cluster per tile, shape by
    // oz_shape); 256 x 256 for N <= 256
    int shape = cols > 256 ? 0 : 1;
    {
        const char *pe0 = getenv("PDL_OZ2_PERSIST");
        if ((pe0 && !strcmp(pe0, "0")) || getenv("PDL_OZ_SHAPE") || getenv("PDL_OZ_NSUB")) shape = oz_shape(rows, cols);
    }
    // persistent 256 x 512 tiles by default (PDL_OZ2_PERSIST=0: one cluster per tile)
    const char *pe = getenv("PDL_OZ2_PERSIST");
    const bool persist = shape == 0 && !(pe && !strcmp(pe, "0"));
    int pclusters = 0;
    const char *he = getenv("PDL_OZ2_HINTS");
    const int hints = he ? atoi(he) : 0;
    if (persist) {
        e0 = oz2_worker_clusters(&pclusters);
        if (e0 != cudaSuccess) return e0;
    }
    int nl = P.n;
    if (persist) {
        nl = oz2_launches_per_chunk(P.n, rows, cols, pclusters);
        if (const char *me = getenv("PDL_OZ2_MERGE")) nl = (P.n + std::max(1, atoi(me)) - 1) / std::max(1, atoi(me));
        nl = std::max(1, std::min(P.n, nl));
    }
    using CF2 = Cfg<2, 1>;
    const int tiles_m2 = (int)((rows + 2 * BM - 1) / (2 * BM)), tiles_n2 = (int)((cols + CF2::BN - 1) / CF2::BN);
    const bool merge = persist && nl < P.n;
    for (int c = 0; c < P.nch && merge; ++c) {
        for (int l = 0; l < nl; ++l) {
            const int t0 = l * P.n / nl, t1 = (l + 1) * P.n / nl, gl = t1 - t0;
            const int64_t off = ((int64_t)c * P.n + t0) * P.Kc;
            CUtensorMap ta, tb;
            if (!map_i8(enc, &ta, A8 + off, (uint64_t)(gl * P.Kc), (uint64_t)rows, (uint64_t)P.ld8, BM) ||
                !map_i8(enc, &tb, Bt8 + off, (uint64_t)(gl * P.Kc), (uint64_t)cols, (uint64_t)P.ld8, BNH))
                return cudaErrorInvalidValue;
            Oz2Moduli mods = {};
            for (int t = 0; t < gl; ++t) {
                const unsigned m = (unsigned)P.m[t0 + t];
                mods.m[t] = (int)m;
                mods.magic[t] = (unsigned)((((unsigned long long)1 << 39) + m - 1) / m);
            }
            const int ncl = std::min(gl * tiles_m2 * tiles_n2, pclusters);
            oz2_gemm_persistent_kernel<2><<<2 * ncl, CF2::THREADS, CF2::SMEM_BYTES, stream>>>(
                ta, tb, R + ((int64_t)c * P.n + t0) * plane, ldr, plane, (int)rows, (int)cols, (int)P.Kc, tiles_m2,
                tiles_n2, group_for_k(P.Kc), gl, mods, hints);
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return e;
            if (launches) ++*launches;
        }
    }
    for (int c = 0; c < P.nch && !merge; ++c) {
        for (int t = 0; t < P.n; ++t) {
            const int64_t off = ((int64_t)c * P.n + t) * P.Kc;
            CUtensorMap ta, tb;
            if (!map_i8(enc, &ta, A8 + off, (uint64_t)P.Kc, (uint64_t)rows, (uint64_t)P.ld8, BM) ||
                !map_i8(enc, &tb, Bt8 + off, (uint64_t)P.Kc, (uint64_t)cols, (uint64_t)P.ld8, BNH))
                return cudaErrorInvalidValue;
            uint8_t *Rp = R + ((int64_t)c * P.n + t) * plane;
            // ceil(2^39 / m): the exact division-by-constant multiplier of the epilogue
            const unsigned magic = (unsigned)((((unsigned long long)1 << 39) + (unsigned)P.m[t] - 1) / (unsigned)P.m[t]);
            if (persist) {
                using CF = Cfg<2, 1>;
                const int tiles_m = (int)((rows + 2 * BM - 1) / (2 * BM)), tiles_n = (int)((cols + CF::BN - 1) / CF::BN);
                const int ncl = std::min(tiles_m * tiles_n, pclusters);
                Oz2Moduli one = {};
                one.m[0] = P.m[t];
                one.magic[0] = magic;
                oz2_gemm_persistent_kernel<2><<<2 * ncl, CF::THREADS, CF::SMEM_BYTES, stream>>>(
                    ta, tb, Rp, ldr, plane, (int)rows, (int)cols, (int)P.Kc, tiles_m, tiles_n, group_for_k(P.Kc), 1,
                    one, hints);
            } else {
                oz_launch<uint8_t>(shape, ta, tb, Rp, ldr, rows, cols, P.Kc, nullptr, nullptr, 0, 0, 1, P.m[t], magic,
                                   stream);
            }
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return e;
            if (launches) ++*launches;
        }
    }
    return cudaSuccess;
}

}  // namespace pdlk
