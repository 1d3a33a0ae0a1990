// k_tf32_2sm.cu -- K2 v3: 3xTF32 tile kernel on a CTA pair (tcgen05 cta_group::2).
//
// Same product as K2 v1 (k_tf32.cu; FP32 task variant, 3xTF32 split from K3,
// K-chunk promotion of the truncating TMEM accumulation, R16) with
// the B200's paired-SM tensor-core mode:
//  * a cluster of 2 CTAs on one TPC computes a 256 x 256 tile: CTA r holds rows
//    [128r, 128r+128) of A and rows [128r, 128r+128) of B^T (half of N) in its
//    own shared memory; the leader CTA issues one
//    tcgen05.mma.cta_group::2.kind::tf32 (M = 256, N = 256, K = 8) that reads
//    the operands of both CTAs and writes each CTA's 128 x 256 FP32
//    accumulator into that CTA's TMEM.  Per SM the tensor core reads half the
//    shared-memory bytes of the 1-SM 128 x 256 shape and L2 traffic halves
//    relative to 128 x 128 tiles;
//  * both CTAs' TMA loads (.cta_group::2) complete on the leader's full
//    barrier; MMA completion is multicast (tcgen05.commit ... multicast) to
//    both CTAs' empty / accumulator-ready barriers; the peer's epilogue warps
//    release accumulator buffers on the leader's barrier through mapa;
//  * TMEM: 512 columns = 2 accumulator buffers x 256; 16 epilogue warps (4 per
//    TMEM lane quarter, 64 columns each) promote every 128-wide K chunk into
//    FP32 registers with round-to-nearest.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"
#include "ptx.cuh"
#include "tcgen05.cuh"

namespace pdlk {

namespace k2x {
constexpr int BM = 128;                 // A rows per CTA (UMMA M = 256 over the pair)
constexpr int BN = 256;                 // UMMA N (cluster tile columns)
constexpr int BNH = BN / 2;             // B^T rows per CTA
constexpr int UMMA_K = 8;
constexpr int EPI_WARPS = 16;
constexpr int EPI_COLS = BN / (EPI_WARPS / 4);           // 64 columns per epilogue warp
constexpr int FIRST_EPI_WARP = 2;   // warps 2..17: each TMEM lane quarter (warp % 4) gets 4 warps
constexpr int THREADS = (FIRST_EPI_WARP + EPI_WARPS) * 32;
constexpr int TMEM_COLS = 512;
constexpr int KCHUNK = 128;             // K chunk promoted from TMEM (R16)
// cluster-tile rows per raster group (r2 sweeps at C4): tf32bf16 8 (DRAM 49.7 -> 36.6 GB per
// launch, higher power-capped clock), 3xtf32 4 (ncu DRAM 54 GB at 4 vs 67 GB at 8)
constexpr int GROUP_M_MIX = 8, GROUP_M_3X = 4;
// K-block width BKF (floats per stage row): 32 = one 128-byte swizzle row (SWIZZLE_128B),
// 3-stage ring of 64 KiB (default); 16 = 64-byte rows (SWIZZLE_64B), 7-stage ring of 32 KiB,
// which keeps 6 stages in flight ahead of the MMAs instead of 2.  The deeper ring measured
// slower (profiles/r02_k2_measurements.md): its smaller stages double the barrier round trips
// and the MMAs lose more than the feed (16.3 TB/s, held back by L2 misses) gains.
template <int BKF>
struct Cfg {
    static constexpr int BK = BKF;
    static constexpr int A_BYTES = BM * BKF * 4;
    static constexpr int B_BYTES = BNH * BKF * 4;
    static constexpr int STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES;
    static constexpr int STAGES = BKF == 32 ? 3 : 7;
    static constexpr int KCB = KCHUNK / BKF;
    static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 + 256;
};
}  // namespace k2x

// UMMA descriptor of a K-major operand tile with BKF-float rows (SW128 or SW64)
template <int BKF>
__device__ __forceinline__ uint64_t k2_desc(uint32_t saddr) {
    if constexpr (BKF == 32) return umma_desc_k_sw128(saddr);
    else return umma_desc_k_sw64(saddr);
}

// MIX = tf32bf16 (R22), BKF = K-block width of the TMA ring (see k2x::Cfg).  The MMA
// order is fixed per 16-wide K step -- MIX: a_lo'*b_hi', a_hi'*b_lo' (kind::f16), then
// a_hi*b_hi for k and k+8 (kind::tf32); 3xTF32: per 8-wide step lo*hi, hi*lo, hi*hi --
// so every BKF (and K2 v1) accumulates in the same order: bitwise the same C.
template <bool MIX, int BKF>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(k2x::THREADS, 1)
    gemm_3xtf32_2sm_kernel(const __grid_constant__ CUtensorMap tAh, const __grid_constant__ CUtensorMap tAl,
                           const __grid_constant__ CUtensorMap tBh, const __grid_constant__ CUtensorMap tBl,
                           float *__restrict__ C, int64_t ldc, int M, int N, int Kp, int tiles_m, int tiles_n,
                           int group_m, int vec_ok, int *dyn_next, int *dyn_mine, int dbg) {
    using namespace k2x;
    using G = Cfg<BKF>;
    constexpr int BK = G::BK, STAGES = G::STAGES, A_BYTES = G::A_BYTES, B_BYTES = G::B_BYTES;
    constexpr int STAGE_BYTES = G::STAGE_BYTES, KCB = G::KCB;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t base = (smem_u32(smem_raw) + 1023u) & ~1023u;
    const uint32_t bar_full = base + STAGES * STAGE_BYTES;   // STAGES x 8 (used in the leader)
    const uint32_t bar_empty = bar_full + STAGES * 8;         // STAGES x 8 (both CTAs)
    const uint32_t bar_tfull = bar_empty + STAGES * 8;        // 2 x 8 (both CTAs)
    const uint32_t bar_tempty = bar_tfull + 16;               // 2 x 8 (leader: both CTAs' epilogues)
    const uint32_t tmem_slot = bar_tempty + 16;
    uint8_t *const gbase = smem_raw + (base - smem_u32(smem_raw));
    volatile uint32_t *tmem_slot_ptr = reinterpret_cast<volatile uint32_t *>(gbase + (tmem_slot - base));

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = cluster_ctarank();

    // grouped raster over 256 x 256 cluster tiles; DYNAMIC: the pair claims its
    // raster index from the counter all Workers share (pairs left over exit)
    int cid = blockIdx.x >> 1;
    if (dyn_next) {
        cid = cluster_claim_tile(dyn_next, dyn_mine, tiles_m * tiles_n);
        if (cid >= tiles_m * tiles_n) return;
    }
    int tm, tn;
    raster_tile(cid, tiles_m, tiles_n, group_m, &tm, &tn);
    const int m0 = tm * (2 * BM) + (int)rank * BM;   // this CTA's A rows
    const int nb0 = tn * BN + (int)rank * BNH;       // this CTA's B^T rows

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(bar_full + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(bar_tfull + 8 * b, 1);
            mbar_init(bar_tempty + 8 * b, 2 * EPI_WARPS);
        }
        fence_barrier_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(tmem_slot),
                     "n"(TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync_all();   // barrier inits and TMEM allocation visible to both CTAs
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem_base = *tmem_slot_ptr;

    const int nk = Kp / BK;
    const int nchunks = (nk + KCB - 1) / KCB;

    if (warp == 0) {
        // ---------------- TMA producer (both CTAs) ----------------
        if (lane == 0) {
            tma_prefetch_desc(&tAh);
            tma_prefetch_desc(&tAl);
            tma_prefetch_desc(&tBh);
            tma_prefetch_desc(&tBl);
            for (int kb = 0; kb < (dbg == 4 ? 0 : nk); ++kb) {
                const int s = kb % STAGES;
                const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
                mbar_wait(bar_empty + 8 * s, ph ^ 1u);
                const uint32_t fb_leader = mapa_shared(bar_full + 8 * s, 0);
                if (dbg == 2 || dbg == 3) {   // measurement only: no operand traffic (PDL_K2_DEBUG=2, 3)
                    if (rank == 0) mbar_arrive(bar_full + 8 * s);
                    continue;
                }
                // PDL_K2_DEBUG=5 (measurement only): the B lo plane is not loaded (a 25 % smaller feed)
                if (rank == 0) mbar_arrive_expect_tx(bar_full + 8 * s, 2 * (STAGE_BYTES - (dbg == 5 ? B_BYTES : 0)));
                const uint32_t st = base + s * STAGE_BYTES;
                const int kl = kb * (MIX ? 2 * BK : BK);   // bf16 [hi' | lo'] rows: 2 BK halves per block
                tma_load_2d_2sm(st, &tAh, fb_leader, kb * BK, m0);
                tma_load_2d_2sm(st + A_BYTES, &tAl, fb_leader, kl, m0);
                tma_load_2d_2sm(st + 2 * A_BYTES, &tBh, fb_leader, kb * BK, nb0);
                if (dbg != 5) tma_load_2d_2sm(st + 2 * A_BYTES + B_BYTES, &tBl, fb_leader, kl, nb0);
            }
        }
    } else if (warp == 1) {
        // ---------------- MMA issuer (leader CTA, one thread) ----------------
        if (rank == 0 && lane == 0) {
            constexpr uint32_t idesc = idesc_tf32(2 * BM, BN);
            constexpr uint32_t idesc16 = idesc_bf16(2 * BM, BN);
            for (int kb = 0; kb < nk; ++kb) {
                const int chunk = kb / KCB, kin = kb - chunk * KCB;
                const uint32_t buf = (uint32_t)chunk & 1u;
                const uint32_t dtm = tmem_base + buf * BN;
                if (kin == 0) {
                    mbar_wait(bar_tempty + 8 * buf, ((uint32_t)(chunk >> 1) & 1u) ^ 1u);
                    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                }
                const int s = kb % STAGES;
                const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
                if (dbg != 4) mbar_wait(bar_full + 8 * s, ph);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const uint32_t st = base + s * STAGE_BYTES;
                const uint32_t ah = st, al = st + A_BYTES, bh = st + 2 * A_BYTES, bl = bh + B_BYTES;
                if (dbg == 1) {   // measurement only: no MMAs, the TMA ring alone (PDL_K2_DEBUG=1)
                } else if constexpr (MIX) {
                    // per 16-wide K step: the BF16 plane holds [hi'(16) | lo'(16)] = 64 bytes
#pragma unroll
                    for (int k16 = 0; k16 < BK / 16; ++k16) {
                        // 64 bytes per 16-wide step in both planes: bf16 [hi' | lo'], tf32 hi (k, k + 8)
                        const uint32_t o = k16 * 64;
                        const uint32_t acc0 = (kin == 0 && k16 == 0) ? 0u : 1u;
                        umma_bf16_2sm(dtm, k2_desc<BKF>(al + o + 32), k2_desc<BKF>(bl + o), idesc16, acc0);
                        umma_bf16_2sm(dtm, k2_desc<BKF>(al + o), k2_desc<BKF>(bl + o + 32), idesc16, 1u);
                        umma_tf32_2sm(dtm, k2_desc<BKF>(ah + o), k2_desc<BKF>(bh + o), idesc, 1u);
                        umma_tf32_2sm(dtm, k2_desc<BKF>(ah + o + 32), k2_desc<BKF>(bh + o + 32), idesc, 1u);
                    }
                } else {
#pragma unroll
                    for (int kk = 0; kk < BK / UMMA_K; ++kk) {
                        const uint32_t off = kk * UMMA_K * 4;
                        const uint32_t acc0 = (kin == 0 && kk == 0) ? 0u : 1u;
                        umma_tf32_2sm(dtm, k2_desc<BKF>(al + off), k2_desc<BKF>(bh + off), idesc, acc0);
                        umma_tf32_2sm(dtm, k2_desc<BKF>(ah + off), k2_desc<BKF>(bl + off), idesc, 1u);
                        umma_tf32_2sm(dtm, k2_desc<BKF>(ah + off), k2_desc<BKF>(bh + off), idesc, 1u);
                    }
                }
                if (dbg != 4) umma_commit_2sm(bar_empty + 8 * s);   // 4: MMAs only, no stage barriers
                if (kin == KCB - 1 || kb == nk - 1) umma_commit_2sm(bar_tfull + 8 * buf);
            }
        }
        __syncwarp();
    } else if (warp >= FIRST_EPI_WARP) {
        // ---------------- epilogue: promote chunks (both CTAs) ----------------
        const int e = warp - FIRST_EPI_WARP;
        const int q = warp & 3;                      // TMEM lane quarter accessible to this warp
        const int cg = e >> 2;                       // column group
        const uint32_t tl = tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(cg * EPI_COLS);
        const uint32_t tempty_leader0 = mapa_shared(bar_tempty, 0);
        float acc[EPI_COLS];
#pragma unroll
        for (int j = 0; j < EPI_COLS; ++j) acc[j] = 0.0f;
        for (int chunk = 0; chunk < nchunks; ++chunk) {
            const uint32_t buf = (uint32_t)chunk & 1u;
            mbar_wait(bar_tfull + 8 * buf, (uint32_t)(chunk >> 1) & 1u);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            if (dbg < 3) {   // PDL_K2_DEBUG=3 (measurement only): chunks are not promoted
#pragma unroll
                for (int c0 = 0; c0 < EPI_COLS; c0 += 16) {
                    uint32_t r[16];
                    tmem_ld16(tl + buf * BN + c0, r);
#pragma unroll
                    for (int j = 0; j < 16; ++j) acc[c0 + j] += __uint_as_float(r[j]);
                }
            }
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
            __syncwarp();
            if (lane == 0) mbar_arrive_cluster(tempty_leader0 + 8 * buf);
        }
        const int row = tm * (2 * BM) + (int)rank * BM + q * 32 + lane;
        const int cbase = tn * BN + cg * EPI_COLS;
        if (row < M) {
            float *crow = C + (int64_t)row * ldc + cbase;
            if (vec_ok && cbase + EPI_COLS <= N) {
#pragma unroll
                for (int j = 0; j < EPI_COLS; j += 4)
                    __stcs(reinterpret_cast<float4 *>(crow + j), make_float4(acc[j], acc[j + 1], acc[j + 2], acc[j + 3]));
            } else {
#pragma unroll
                for (int j = 0; j < EPI_COLS; ++j)
                    if (cbase + j < N) crow[j] = acc[j];
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    cluster_sync_all();   // both CTAs done with TMEM and with each other's shared memory
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(TMEM_COLS));
    }
}

// bf16 = 1: the bf16 [hi' | lo'] plane of the TF32+BF16 split (2 Kp halves per row).
// Box rows of BKF floats = BKF * 4 bytes either way.
static bool map_f32_2sm(EncodeTiledFn enc, CUtensorMap *m, const float *ptr, uint64_t Kp, uint64_t rows,
                        uint32_t box_rows, uint64_t ld, int bf16, int bkf) {
    cuuint64_t dims[2] = {bf16 ? 2 * Kp : Kp, rows};
    cuuint64_t strides[1] = {(ld ? ld : Kp) * 4};
    cuuint32_t box[2] = {(cuuint32_t)(bf16 ? 2 * bkf : bkf), box_rows};
    cuuint32_t es[2] = {1, 1};
    return enc(m, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
               const_cast<float *>(ptr), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               bkf == 32 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// K-block width of the CTA-pair kernel: PDL_K2_BK = 16 | 32 (measurement knob),
// default 32: the 7-stage SW64 ring measured slower at C4 (tf32bf16 29.8 vs 23.9 ms,
// 3xtf32 33.1 vs 32.1 ms; r2s19), so a deeper prefetch is not what the kernel lacks.
// Both give bitwise the same C.
static int k2_bkf() {
    const char *e = getenv("PDL_K2_BK");
    return (e && atoi(e) == 16) ? 16 : 32;
}

template <bool MIX, int BKF>
static cudaError_t launch_k2x(const CUtensorMap &tah, const CUtensorMap &tal, const CUtensorMap &tbh,
                              const CUtensorMap &tbl, float *C, int64_t ldc, int64_t M, int64_t N, int64_t Kp,
                              cudaStream_t stream, int *dyn_next, int *dyn_mine) {
    using namespace k2x;
    auto kern = gemm_3xtf32_2sm_kernel<MIX, BKF>;
    // measurement knob (C is garbage): 1 = TMA ring only, 2 = MMAs only, 3 = MMAs only, no chunk promotion,
    // 4 = MMAs only without the per-stage full / empty barriers
    const char *de = getenv("PDL_K2_DEBUG");
    const int dbg = de ? atoi(de) : 0;
    constexpr int SMEM = Cfg<BKF>::SMEM_BYTES;
    int dev = 0;
    cudaGetDevice(&dev);
    static bool attr_done[64] = {};
    if (dev < 64 && !attr_done[dev]) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
        if (e != cudaSuccess) return e;
        attr_done[dev] = true;
    }
    const int tiles_m = (int)((M + 2 * BM - 1) / (2 * BM)), tiles_n = (int)((N + BN - 1) / BN);
    const int vec_ok = ((reinterpret_cast<uintptr_t>(C) & 15u) == 0 && (ldc & 3) == 0) ? 1 : 0;
    kern<<<2 * tiles_m * tiles_n, THREADS, SMEM, stream>>>(tah, tal, tbh, tbl, C, ldc, (int)M, (int)N, (int)Kp,
                                                          tiles_m, tiles_n, raster_group_m(MIX ? GROUP_M_MIX : GROUP_M_3X), vec_ok,
                                                          dyn_next, dyn_mine, dbg);
    return cudaGetLastError();
}

cudaError_t launch_gemm_3xtf32_2sm(EncodeTiledFn enc, const float *Ahi, const float *Alo, const float *Bhi,
                                   const float *Blo, int64_t Kp, float *C, int64_t ldc, int64_t M, int64_t N,
                                   cudaStream_t stream, int *dyn_next, int *dyn_mine, int64_t lda_s, int mix) {
    using namespace k2x;
    if (M <= 0 || N <= 0 || Kp <= 0) return cudaSuccess;
    const int bkf = k2_bkf();
    CUtensorMap tah, tal, tbh, tbl;
    if (!map_f32_2sm(enc, &tah, Ahi, Kp, M, BM, lda_s, 0, bkf) || !map_f32_2sm(enc, &tal, Alo, Kp, M, BM, lda_s, mix, bkf) ||
        !map_f32_2sm(enc, &tbh, Bhi, Kp, N, BNH, 0, 0, bkf) || !map_f32_2sm(enc, &tbl, Blo, Kp, N, BNH, 0, mix, bkf))
        return cudaErrorInvalidValue;
    if (bkf == 32)
        return mix ? launch_k2x<true, 32>(tah, tal, tbh, tbl, C, ldc, M, N, Kp, stream, dyn_next, dyn_mine)
                   : launch_k2x<false, 32>(tah, tal, tbh, tbl, C, ldc, M, N, Kp, stream, dyn_next, dyn_mine);
    return mix ? launch_k2x<true, 16>(tah, tal, tbh, tbl, C, ldc, M, N, Kp, stream, dyn_next, dyn_mine)
               : launch_k2x<false, 16>(tah, tal, tbh, tbl, C, ldc, M, N, Kp, stream, dyn_next, dyn_mine);
}

}  // namespace pdlk
