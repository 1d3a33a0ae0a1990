// k_tf32.cu -- K3 (TF32 hi/lo split) and K2 (3xTF32 tile kernel on tcgen05).
//
// FP32 variant of the DGEMM task (same task interface, L1032-1039; the paper's
// own task is FP64, L1402-1406; the FP32 variant follows the north star's
// "if inputs are FP32, use split-TF32/3xTF32 ... so accuracy holds").
//
// Split (K3): x = hi + lo + r with hi = rna_tf32(x), lo = rna_tf32(x - hi)
// (x - hi is exact in fp32), |r| <= 2^-22 |x|.  Product (K2):
//   a*b ~= a_lo*b_hi + a_hi*b_lo + a_hi*b_hi     (a_lo*b_lo, ~2^-22, dropped)
// The split is a pre-pass that also transposes B to K-major, so both UMMA
// operands use the canonical K-major SWIZZLE_128B layout.
//
// K2 (v1, DESIGN.md SS Kernels/K2): CTA tile 128 x 128, BK = 32 fp32 (one
// 128-byte swizzle atom), 3-stage TMA ring of {A_hi, A_lo, B_hi, B_lo};
// warp 0 = TMA producer, warp 1 = TMEM allocator + single-thread tcgen05.mma
// issuer (kind::tf32, M=128, N=128, K=8 per instruction, FP32 accumulator in
// TMEM, 128 columns), warps 2..5 = epilogue (tcgen05.ld 32x32b -> registers
// -> vectorised global stores).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"
#include "ptx.cuh"
#include "tcgen05.cuh"

namespace pdlk {

// ------------------------------------------------------------------------
// K3: split pre-pass
// ------------------------------------------------------------------------
__device__ __forceinline__ float tf32_rna(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}

// bf16 bits of x, round to nearest even
__device__ __forceinline__ uint32_t bf16_rn_bits(float x) {
    uint16_t r;
    asm("cvt.rn.bf16.f32 %0, %1;" : "=h"(r) : "f"(x));
    return r;
}

// Split of 4 consecutive k (k0 % 4 == 0) of one row into its K-major outputs.
//  3xTF32 (mix = 0): hi[k] = rna_tf32(x), lo[k] = rna_tf32(x - hi)      (fp32 planes)
//  TF32+BF16 (mix = 1, R22): hi[k] = rna_tf32(x) as before; the second
//  plane holds bf16 pairs per 16-wide K block b: halves [32 b, 32 b + 16) =
//  rn_bf16(hi), [32 b + 16, 32 b + 32) = rn_bf16(x - hi)  (64 bytes per block: one
//  kind::f16 K = 16 step reads 32 of them; the K2 TMA boxes take 1 or 2 blocks)
__device__ __forceinline__ void split_store4(const float (&v)[4], float *hi, float *lo, int64_t k0, int mix) {
    float h[4], l[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
        h[u] = tf32_rna(v[u]);
        l[u] = v[u] - h[u];   // exact in fp32
    }
    *reinterpret_cast<float4 *>(hi + k0) = make_float4(h[0], h[1], h[2], h[3]);
    if (!mix) {
#pragma unroll
        for (int u = 0; u < 4; ++u) l[u] = tf32_rna(l[u]);
        *reinterpret_cast<float4 *>(lo + k0) = make_float4(l[0], l[1], l[2], l[3]);
    } else {
        uint16_t *pl = reinterpret_cast<uint16_t *>(lo) + (k0 >> 4) * 32 + (k0 & 15);
        const uint2 hb = make_uint2(bf16_rn_bits(h[0]) | (bf16_rn_bits(h[1]) << 16),
                                    bf16_rn_bits(h[2]) | (bf16_rn_bits(h[3]) << 16));
        const uint2 lb = make_uint2(bf16_rn_bits(l[0]) | (bf16_rn_bits(l[1]) << 16),
                                    bf16_rn_bits(l[2]) | (bf16_rn_bits(l[3]) << 16));
        *reinterpret_cast<uint2 *>(pl) = hb;
        *reinterpret_cast<uint2 *>(pl + 16) = lb;
    }
}

__global__ void split_rows_kernel(const float *__restrict__ A, int64_t lda, int64_t M, int64_t K,
                                  float *__restrict__ hi, float *__restrict__ lo, int64_t Kp, int64_t ldo, int vec,
                                  int mix) {
    // one thread per 4 consecutive k of one row (Kp % 4 == 0)
    const int64_t q = Kp >> 2;
    const int64_t total = M * q;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = t / q, k0 = (t - i * q) << 2;
        const float *src = A + i * lda;
        float v[4];
        if (vec && k0 + 3 < K) {   // 16-byte aligned rows: one LDG.128
            const float4 x = __ldcs(reinterpret_cast<const float4 *>(src + k0));
            v[0] = x.x, v[1] = x.y, v[2] = x.z, v[3] = x.w;
        } else {
#pragma unroll
            for (int u = 0; u < 4; ++u) v[u] = (k0 + u < K) ? __ldg(src + k0 + u) : 0.0f;
        }
        split_store4(v, hi + i * ldo, lo + i * ldo, k0, mix);
    }
}

// B (K x N) -> B^T split (N x Kp); 64 x 64 tiles through shared memory, 16-byte
// loads along n and 16-byte stores along k (4 of each per thread).  The 32 x 32
// scalar version moved 4 KB per CTA with 4-byte accesses and ran at 48 % of HBM
// (profiles/r01_ncu_prof_k3.json).
__global__ void __launch_bounds__(256) split_cols_t_kernel(const float *__restrict__ B, int64_t ldb, int64_t K,
                                                           int64_t N, float *__restrict__ hi, float *__restrict__ lo,
                                                           int64_t Kp, int vec, int mix) {
    __shared__ float t[64][65];
    const int64_t k0 = (int64_t)blockIdx.y * 64, n0 = (int64_t)blockIdx.x * 64;
    const int cq = threadIdx.x & 15, r0 = threadIdx.x >> 4;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int r = r0 + 16 * i;
        const int64_t k = k0 + r, n = n0 + 4 * cq;
        float v[4];
        if (vec && k < K && n + 3 < N) {
            const float4 x = __ldcs(reinterpret_cast<const float4 *>(B + k * ldb + n));
            v[0] = x.x, v[1] = x.y, v[2] = x.z, v[3] = x.w;
        } else {
#pragma unroll
            for (int j = 0; j < 4; ++j) v[j] = (k < K && n + j < N) ? __ldg(B + k * ldb + n + j) : 0.0f;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) t[r][4 * cq + j] = v[j];
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int nr = r0 + 16 * i;
        const int64_t n = n0 + nr, k = k0 + 4 * cq;
        if (n < N && k < Kp) {   // Kp % 32 == 0: a group of 4 k is all inside or all outside
            float v[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) v[j] = t[4 * cq + j][nr];
            split_store4(v, hi + n * Kp, lo + n * Kp, k, mix);
        }
    }
}

cudaError_t launch_split_rows(const float *A, int64_t lda, int64_t M, int64_t K, float *hi, float *lo, int64_t Kp,
                              cudaStream_t s, int64_t ldo, int mix) {
    if (ldo <= 0) ldo = Kp;
    if (M <= 0 || Kp <= 0) return cudaSuccess;
    const int64_t total = M * (Kp >> 2);
    int blocks = (int)((total + 255) / 256);
    if (blocks > 148 * 16) blocks = 148 * 16;
    const int vec = ((reinterpret_cast<uintptr_t>(A) & 15u) == 0 && (lda & 3) == 0) ? 1 : 0;
    split_rows_kernel<<<blocks, 256, 0, s>>>(A, lda, M, K, hi, lo, Kp, ldo, vec, mix);
    return cudaGetLastError();
}

cudaError_t launch_split_cols_t(const float *B, int64_t ldb, int64_t K, int64_t N, float *hi, float *lo, int64_t Kp,
                                cudaStream_t s, int mix) {
    if (N <= 0 || Kp <= 0) return cudaSuccess;
    dim3 grid((unsigned)((N + 63) / 64), (unsigned)((Kp + 63) / 64));
    const int vec = ((reinterpret_cast<uintptr_t>(B) & 15u) == 0 && (ldb & 3) == 0) ? 1 : 0;
    split_cols_t_kernel<<<grid, 256, 0, s>>>(B, ldb, K, N, hi, lo, Kp, vec, mix);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------
// K2: 3xTF32 tcgen05 GEMM
// ------------------------------------------------------------------------
namespace k2 {
constexpr int BM = 128, BN = 128, BK = K2_BK, STAGES = 3;
constexpr int UMMA_K = 8;                           // tf32: 32 bytes of K per instruction
constexpr int A_BYTES = BM * BK * 4;                // 16 KiB
constexpr int B_BYTES = BN * BK * 4;                // 16 KiB
constexpr int STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES;   // hi + lo of both operands
constexpr int EPI_WARPS = 4;
constexpr int THREADS = (2 + EPI_WARPS) * 32;
constexpr int TMEM_COLS = 2 * BN;                   // double-buffered FP32 accumulator
// K-chunk promotion (R16): the tensor cores accumulate a chunk of
// KCB k-blocks (KCB*BK = 128 of K) in TMEM; the epilogue warps add each chunk
// sum into an FP32 register accumulator with round-to-nearest while the MMA
// warp fills the other TMEM buffer.  Measured on the B200 the TMEM
// accumulation truncates (mean signed error -1.0e-8 * K for U[0,1) inputs),
// so without promotion K >= 1024 breaks the 1e-5 bar.
constexpr int KCB = 4;
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 + 256;
}  // namespace k2

template <bool MIX>
__global__ void __launch_bounds__(k2::THREADS, 1)
    gemm_3xtf32_kernel(const __grid_constant__ CUtensorMap tAh, const __grid_constant__ CUtensorMap tAl,
                       const __grid_constant__ CUtensorMap tBh, const __grid_constant__ CUtensorMap tBl,
                       float *__restrict__ C, int64_t ldc, int M, int N, int Kp, int tiles_m, int tiles_n,
                       int vec_ok) {
    using namespace k2;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t base = (smem_u32(smem_raw) + 1023u) & ~1023u;
    const uint32_t bar_full = base + STAGES * STAGE_BYTES;      // STAGES x 8
    const uint32_t bar_empty = bar_full + STAGES * 8;            // STAGES x 8
    const uint32_t bar_tfull = bar_empty + STAGES * 8;           // 2 x 8: accumulator buffer ready
    const uint32_t bar_tempty = bar_tfull + 16;                  // 2 x 8: accumulator buffer drained
    const uint32_t tmem_slot = bar_tempty + 16;                  // 4 bytes
    uint8_t *const gbase = smem_raw + (base - smem_u32(smem_raw));
    volatile uint32_t *tmem_slot_ptr = reinterpret_cast<volatile uint32_t *>(gbase + (tmem_slot - base));

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    // grouped raster (16 tile rows per group)
    const int bid = blockIdx.x;
    const int per_group = 16 * tiles_n;
    const int g = bid / per_group;
    const int first_m = g * 16;
    const int gsz = min(tiles_m - first_m, 16);
    const int tm = first_m + (bid % per_group) % gsz;
    const int tn = (bid % per_group) / gsz;

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(bar_full + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(bar_tfull + 8 * b, 1);
            mbar_init(bar_tempty + 8 * b, EPI_WARPS);
        }
        fence_barrier_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(tmem_slot),
                     "n"(TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem_base = *tmem_slot_ptr;

    const int nk = Kp / BK;
    const int nchunks = (nk + KCB - 1) / KCB;

    if (warp == 0) {
        // ---------------- TMA producer ----------------
        if (lane == 0) {
            tma_prefetch_desc(&tAh);
            tma_prefetch_desc(&tAl);
            tma_prefetch_desc(&tBh);
            tma_prefetch_desc(&tBl);
            const int m0 = tm * BM, n0 = tn * BN;
            for (int kb = 0; kb < nk; ++kb) {
                const int s = kb % STAGES;
                const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
                mbar_wait(bar_empty + 8 * s, ph ^ 1u);
                const uint32_t fb = bar_full + 8 * s;
                mbar_arrive_expect_tx(fb, STAGE_BYTES);
                const uint32_t st = base + s * STAGE_BYTES;
                tma_load_2d(st, &tAh, fb, kb * BK, m0);
                const int kl = kb * (MIX ? 2 * BK : BK);   // bf16 [hi' | lo'] rows: 64 halves per block
                tma_load_2d(st + A_BYTES, &tAl, fb, kl, m0);
                tma_load_2d(st + 2 * A_BYTES, &tBh, fb, kb * BK, n0);
                tma_load_2d(st + 2 * A_BYTES + B_BYTES, &tBl, fb, kl, n0);
            }
        }
    } else if (warp == 1) {
        // ---------------- MMA issuer (one thread) ----------------
        if (lane == 0) {
            constexpr uint32_t idesc = idesc_tf32(BM, BN);
            for (int kb = 0; kb < nk; ++kb) {
                const int chunk = kb / KCB, kin = kb - chunk * KCB;
                const uint32_t buf = (uint32_t)chunk & 1u;
                const uint32_t dtm = tmem_base + buf * BN;
                if (kin == 0) {
                    // wait until the epilogue drained this accumulator buffer (2 chunks ago)
                    mbar_wait(bar_tempty + 8 * buf, ((uint32_t)(chunk >> 1) & 1u) ^ 1u);
                    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                }
                const int s = kb % STAGES;
                const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
                mbar_wait(bar_full + 8 * s, ph);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const uint32_t st = base + s * STAGE_BYTES;
                const uint32_t ah = st, al = st + A_BYTES, bh = st + 2 * A_BYTES, bl = bh + B_BYTES;
                if constexpr (MIX) {
                    // TF32+BF16 (R22), per 16-wide K step (the order of K2 v3): the two
                    // correction products as kind::f16 on the bf16 [hi'(16) | lo'(16)]
                    // blocks (K = 16 = 32 B per instruction), then hi*hi in TF32 for k, k + 8
                    constexpr uint32_t idesc16 = idesc_bf16(BM, BN);
#pragma unroll
                    for (int k16 = 0; k16 < BK / 16; ++k16) {
                        const uint32_t o = k16 * 64;
                        const uint32_t acc0 = (kin == 0 && k16 == 0) ? 0u : 1u;
                        umma_bf16(dtm, umma_desc_k_sw128(al + o + 32), umma_desc_k_sw128(bl + o), idesc16, acc0);
                        umma_bf16(dtm, umma_desc_k_sw128(al + o), umma_desc_k_sw128(bl + o + 32), idesc16, 1u);
                        umma_tf32(dtm, umma_desc_k_sw128(ah + o), umma_desc_k_sw128(bh + o), idesc, 1u);
                        umma_tf32(dtm, umma_desc_k_sw128(ah + o + 32), umma_desc_k_sw128(bh + o + 32), idesc, 1u);
                    }
                } else {
#pragma unroll
                    for (int kk = 0; kk < BK / UMMA_K; ++kk) {
                        const uint32_t off = kk * UMMA_K * 4;   // 32 B per K step inside the swizzle atom
                        const uint32_t acc0 = (kin == 0 && kk == 0) ? 0u : 1u;
                        // small terms first: lo*hi, hi*lo, then hi*hi
                        umma_tf32(dtm, umma_desc_k_sw128(al + off), umma_desc_k_sw128(bh + off), idesc, acc0);
                        umma_tf32(dtm, umma_desc_k_sw128(ah + off), umma_desc_k_sw128(bl + off), idesc, 1u);
                        umma_tf32(dtm, umma_desc_k_sw128(ah + off), umma_desc_k_sw128(bh + off), idesc, 1u);
                    }
                }
                umma_commit(bar_empty + 8 * s);                 // smem stage free when these MMAs finish
                if (kin == KCB - 1 || kb == nk - 1) umma_commit(bar_tfull + 8 * buf);   // chunk sum ready
            }
        }
        __syncwarp();
    } else {
        // ---------------- epilogue warps 2..5: promote chunks, then store ----------------
        const int q = warp & 3;                         // TMEM lane quarter of this warp
        const uint32_t tl = tmem_base + ((uint32_t)(q * 32) << 16);
        float acc[BN];
#pragma unroll
        for (int j = 0; j < BN; ++j) acc[j] = 0.0f;
        for (int chunk = 0; chunk < nchunks; ++chunk) {
            const uint32_t buf = (uint32_t)chunk & 1u;
            mbar_wait(bar_tfull + 8 * buf, (uint32_t)(chunk >> 1) & 1u);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
            for (int c0 = 0; c0 < BN; c0 += 32) {
                uint32_t r[32];
                tmem_ld32(tl + buf * BN + c0, r);
#pragma unroll
                for (int j = 0; j < 32; ++j) acc[c0 + j] += __uint_as_float(r[j]);   // RN fp32 promotion
            }
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
            __syncwarp();
            if (lane == 0) mbar_arrive(bar_tempty + 8 * buf);
        }
        const int row = tm * BM + q * 32 + lane;
        if (row < M) {
            float *crow = C + (int64_t)row * ldc + (int64_t)tn * BN;
            const int cbase = tn * BN;
            if (vec_ok && cbase + BN <= N) {
#pragma unroll
                for (int j = 0; j < BN; j += 4)
                    *reinterpret_cast<float4 *>(crow + j) = make_float4(acc[j], acc[j + 1], acc[j + 2], acc[j + 3]);
            } else {
#pragma unroll
                for (int j = 0; j < BN; ++j)
                    if (cbase + j < N) crow[j] = acc[j];
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(TMEM_COLS));
    }
}

// bf16 = 1: the plane holds the bf16 [hi' | lo'] rows of the TF32+BF16 split (2 Kp
// halves per row, boxes of 64 halves = the same 128 bytes per K block)
static bool map_f32(EncodeTiledFn enc, CUtensorMap *m, const float *ptr, uint64_t Kp, uint64_t rows, uint32_t box_rows,
                    uint64_t ld = 0, int bf16 = 0) {
    cuuint64_t dims[2] = {bf16 ? 2 * Kp : Kp, rows};
    cuuint64_t strides[1] = {(ld ? ld : Kp) * 4};
    cuuint32_t box[2] = {(cuuint32_t)(bf16 ? 2 * k2::BK : k2::BK), box_rows};
    cuuint32_t es[2] = {1, 1};
    return enc(m, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float *>(ptr),
               dims, strides, box, es,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

cudaError_t launch_gemm_3xtf32(EncodeTiledFn enc, const float *Ahi, const float *Alo, const float *Bhi,
                               const float *Blo, int64_t Kp, float *C, int64_t ldc, int64_t M, int64_t N,
                               cudaStream_t stream, int64_t lda_s, int mix) {
    using namespace k2;
    if (M <= 0 || N <= 0 || Kp <= 0) return cudaSuccess;
    CUtensorMap tah, tal, tbh, tbl;
    if (!map_f32(enc, &tah, Ahi, Kp, M, BM, lda_s) || !map_f32(enc, &tal, Alo, Kp, M, BM, lda_s, mix) ||
        !map_f32(enc, &tbh, Bhi, Kp, N, BN) || !map_f32(enc, &tbl, Blo, Kp, N, BN, 0, mix))
        return cudaErrorInvalidValue;
    int dev = 0;
    cudaGetDevice(&dev);
    static bool attr_done[2][64] = {};
    if (dev < 64 && !attr_done[mix ? 1 : 0][dev]) {
        cudaError_t e = cudaFuncSetAttribute(mix ? gemm_3xtf32_kernel<true> : gemm_3xtf32_kernel<false>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
        if (e != cudaSuccess) return e;
        attr_done[mix ? 1 : 0][dev] = true;
    }
    const int tiles_m = (int)((M + BM - 1) / BM), tiles_n = (int)((N + BN - 1) / BN);
    const int vec_ok = ((reinterpret_cast<uintptr_t>(C) & 15u) == 0 && (ldc & 3) == 0) ? 1 : 0;
    (mix ? gemm_3xtf32_kernel<true> : gemm_3xtf32_kernel<false>)<<<tiles_m * tiles_n, THREADS, SMEM_BYTES, stream>>>(
        tah, tal, tbh, tbl, C, ldc, (int)M, (int)N, (int)Kp, tiles_m, tiles_n, vec_ok);
    return cudaGetLastError();
}

}  // namespace pdlk
