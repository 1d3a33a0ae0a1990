// k_dgemm.cu -- K1: FP64 tile-task kernel for sm_100a.
//
// Computes one Worker's C rectangle, C[rows x cols] = A[rows x K] * B[K x cols]
// in double precision: the paper's case-study task, "double precision matrix
// multiplication ... (DGEMM)" (PAPER.md SS IV-D, L1402-1406), executed there
// by CUBLAS DGEMM on the GPU Workers (L1428-1431).  All tile tasks of the
// Worker's BLOCK rectangle are coalesced into one launch (K1).
//
// B200 design (DESIGN.md SS Kernels/K1):
//  * FP64 tensor cores: `mma.sync.m8n8k4.f64` -> SASS DMMA.8x8x4 (tcgen05 has
//    no f64 kind on sm_100a).  DMMA runs at the chip's FP64 rate (64 FMA/clk/SM).
//  * Operands staged by TMA (cp.async.bulk.tensor, SWIZZLE_128B) into a
//    4-stage shared-memory ring; mbarrier full/empty handshakes; eight DMMA
//    warps (warp tile 64 x 32, 128 accumulator registers/thread), thread 0
//    refilling each stage once all warps released it.
//  * Bank-conflict-free 16-byte fragment loads (ld.shared.v2.f64): within
//    each 16-wide K block the four k4 MMA steps take k = {0,4,10,14},
//    {1,5,11,15}, {2,6,8,12}, {3,7,9,13} (same permutation for A and B); with
//    the 128B swizzle every quarter-warp hits 8 distinct bank groups, and one
//    A load serves two steps, one B load two n8 tiles.  Fragments of the next
//    step (and next K block) are prefetched before the current DMMAs.  The summation
//    order per C element is fixed by this kernel alone, so results do not
//    depend on the Worker rectangle or task tile (bitwise invariance, pin P7).
//  * CTA tile 128 x 128, grouped rasterisation for L2 reuse, masked
//    vectorised (16 B) epilogue straight from the accumulators.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "kernels.h"
#include "ptx.cuh"

namespace pdlk {

namespace k1 {
// Two CTA shapes with the same warp tile (64 x 32) and the same per-element
// summation order, so they give bitwise the same C (pin P7): 128 x 128 (eight
// DMMA warps, one CTA per SM) and, for grids too small to fill the 148 SMs,
// 64 x 128 (four warps, two CTAs per SM).
template <int BM_>
struct Shape {
    static constexpr int BM = BM_, BN = 128, BK = 16, STAGES = 4;
    static constexpr int A_BYTES = BM * BK * 8;   // 16 KiB (BM 128) / 8 KiB (BM 64)
    static constexpr int B_BYTES = BK * BN * 8;   // 16 KiB, as BN/16 sub-boxes of 16 x 16 doubles
    static constexpr int B_SUB_BYTES = BK * 16 * 8;
    static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
    static constexpr int NCONS = BM / 16;          // DMMA warps (2 or 1 warp rows x 4); thread 0 also issues TMA
    static constexpr int THREADS = NCONS * 32;     // keeps the 255-register budget per thread
    static constexpr int MIN_CTAS = 128 / BM;      // CTAs per SM
    static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 2 * STAGES * 8 + 1024;
};
constexpr int GROUP_M = 8;             // tile rows per raster group (ncu sweep: 8 -> least DRAM traffic)
}  // namespace k1

// Rate of a 64-row CTA relative to the 128-row CTA's per-SM rate: alone on an
// SM (four DMMA warps) and two per SM (measured, tools/k1_shape_sweep.py).
constexpr double K1_E1 = 0.69, K1_E2 = 0.93;

// 128B-swizzled byte offset of (row, 8-byte column j in [0,16)) inside a
// buffer of 128-byte rows whose base is 1024-byte aligned.
__device__ __forceinline__ uint32_t swz128(uint32_t row, uint32_t j) {
    return row * 128u + ((((j >> 1) ^ (row & 7u)) << 4) | ((j & 1u) << 3));
}

__device__ __forceinline__ void lds128(uint32_t addr, double &x, double &y) {
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(x), "=d"(y) : "r"(addr));
}

__device__ __forceinline__ void dmma(double &c0, double &c1, double a, double b) {
    asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

template <int BM_>
__global__ void __launch_bounds__(k1::Shape<BM_>::THREADS, k1::Shape<BM_>::MIN_CTAS)
    dgemm_k1_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                    double *__restrict__ C, int64_t ldc, int M, int N, int K, int tiles_m, int tiles_n,
                    int group_m, int vec_ok, int *dyn_next, int *dyn_mine, const uint32_t *tile_mask,
                    int64_t ld_mask, const uint32_t *elem_mask, int64_t ld_emask) {
    using S = k1::Shape<BM_>;
    constexpr int BM = S::BM, BN = S::BN, BK = S::BK, STAGES = S::STAGES, NCONS = S::NCONS;
    constexpr int A_BYTES = S::A_BYTES, B_SUB_BYTES = S::B_SUB_BYTES, STAGE_BYTES = S::STAGE_BYTES;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t base = (smem_u32(smem_raw) + 1023u) & ~1023u;
    const uint32_t bar_full = base + STAGES * STAGE_BYTES;
    const uint32_t bar_empty = bar_full + STAGES * 8;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    // grouped raster: group_m tile rows sweep the tile columns together.  Under
    // the DYNAMIC distribution the raster index is claimed from the counter all
    // Workers share instead of taken from blockIdx (CTAs left over exit).
    int bid = blockIdx.x;
    if (dyn_next) {
        bid = cta_claim_tile(dyn_next, dyn_mine, tiles_m * tiles_n);
        if (bid >= tiles_m * tiles_n) return;
    }
    const int per_group = group_m * tiles_n;
    const int g = bid / per_group;
    const int first_m = g * group_m;
    const int gsz = min(tiles_m - first_m, group_m);
    const int tm = first_m + (bid % per_group) % gsz;
    const int tn = (bid % per_group) / gsz;
    // recompute set of the Ozaki-II certificate: other tiles exit untouched
    if (tile_mask && !tile_mask[(int64_t)((tm * BM) >> 7) * ld_mask + ((tn * BN) >> 7)]) return;

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(bar_full + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, NCONS);
        }
        fence_barrier_init();
    }
    __syncthreads();

    const int nk = (K + BK - 1) / BK;

    // ---------------- TMA issue (thread 0) ----------------
    // Prologue fills the ring; afterwards thread 0 refills stage s with
    // k-block kb + STAGES as soon as all eight warps have released it.
    const int m0 = tm * BM, n0 = tn * BN;
    auto issue = [&](int kb) {
        const int s = kb % STAGES;
        const uint32_t fb = bar_full + 8 * s;
        mbar_arrive_expect_tx(fb, STAGE_BYTES);
        const uint32_t sa = base + s * STAGE_BYTES;
        const uint32_t sb = sa + A_BYTES;
        tma_load_2d(sa, &tmA, fb, kb * BK, m0);
#pragma unroll
        for (int j = 0; j < BN / 16; ++j) tma_load_2d(sb + j * B_SUB_BYTES, &tmB, fb, n0 + 16 * j, kb * BK);
    };
    if (threadIdx.x == 0) {
        tma_prefetch_desc(&tmA);
        tma_prefetch_desc(&tmB);
        for (int kb = 0; kb < STAGES && kb < nk; ++kb) issue(kb);
    }

    // ---------------- DMMA consumers ----------------
    // Fragment schedule (K1): each lane reads 16-byte chunks.  A: for
    // row m the lane with MMA-k index p reads chunk cA(p) = {0,2,5,7}[p] (k =
    // 2cA, 2cA+1: steps 0 and 1) and chunk cA(p)^1 (steps 2 and 3).  B: per step
    // one 16 B load per 16-column pair gives the b operand of two n8 tiles
    // (columns 2j and 2j+1).  The k order per 16-wide block is
    // {0,4,10,14},{1,5,11,15},{2,6,8,12},{3,7,9,13}; with the 128B swizzle every
    // quarter-warp of every ld.shared.v2.f64 hits 8 distinct bank groups.
    const int wm = warp >> 2, wn = warp & 3;   // (BM / 64) x 4 warps, warp tile 64 x 32
    const uint32_t g4 = (uint32_t)lane >> 2;   // groupID (MMA row / B column pair)
    const uint32_t p = (uint32_t)lane & 3u;    // thread in group (MMA k index)
    const uint32_t cA = (0x7520u >> (4u * p)) & 0xFu;

    double acc[8][4][2];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;

    const uint32_t rowA = 64u * wm + g4;
    const uint32_t offA0 = rowA * 128u + ((cA ^ g4) << 4);           // + mi*1024, half 0
    const uint32_t offA1 = rowA * 128u + (((cA ^ 1u) ^ g4) << 4);    // half 1
    uint32_t offB[4];
#pragma unroll
    for (int st = 0; st < 4; ++st) {
        const uint32_t k = 2u * (st < 2 ? cA : (cA ^ 1u)) + (uint32_t)(st & 1);
        offB[st] = A_BYTES + (2u * wn) * B_SUB_BYTES + k * 128u + ((g4 ^ (k & 7u)) << 4);
    }

    double a[2][8][2];   // [half][mi][k of the two steps of that half]
    double b[2][4];      // [step parity][ni]
    auto load_a = [&](uint32_t st_base, int half) {
        const uint32_t o = st_base + (half ? offA1 : offA0);
#pragma unroll
        for (int mi = 0; mi < 8; ++mi) lds128(o + mi * 1024u, a[half][mi][0], a[half][mi][1]);
    };
    auto load_b = [&](uint32_t st_base, int st) {
        const uint32_t o = st_base + offB[st];
        lds128(o, b[st & 1][0], b[st & 1][1]);                      // columns 16*pair + 2j, 2j+1, pair 0
        lds128(o + B_SUB_BYTES, b[st & 1][2], b[st & 1][3]);        // pair 1
    };

    if (nk > 0) {
        mbar_wait(bar_full, 0);
        load_a(base, 0);
        load_b(base, 0);
    }
    for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % STAGES;
        const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
        const uint32_t sa = base + s * STAGE_BYTES;
        const int sn = (kb + 1) % STAGES;
        const uint32_t san = base + sn * STAGE_BYTES;
#pragma unroll
        for (int st = 0; st < 4; ++st) {
            // prefetch the operands of the next step (next k-block for st == 3)
            if (st == 0) load_a(sa, 1);
            if (st == 2) {
                if (kb + 1 < nk) mbar_wait(bar_full + 8 * sn, (uint32_t)((kb + 1) / STAGES) & 1u);
                load_a(san, 0);
            }
            if (st < 3) load_b(sa, st + 1);
            else load_b(san, 0);
            const int h = st >> 1, e = st & 1;
#pragma unroll
            for (int mi = 0; mi < 8; ++mi)
#pragma unroll
                for (int ni = 0; ni < 4; ++ni) {
                    // n8 tile ni uses columns 16*(ni>>1) + 2j + (ni&1) of the warp's 32
                    const double bv = b[st & 1][(ni >> 1) * 2 + (ni & 1)];
                    dmma(acc[mi][ni][0], acc[mi][ni][1], a[h][mi][e], bv);
                }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(bar_empty + 8 * s);
        if (threadIdx.x == 0 && kb + STAGES < nk) {
            mbar_wait(bar_empty + 8 * s, ph);
            issue(kb + STAGES);
        }
    }

    // ---------------- epilogue: registers -> global ----------------
    // acc[mi][2q+e][h] is C[row][32wn + 16q + 4p + 2h + e]: each lane owns 4
    // consecutive columns per 16-column pair -> two 16-byte stores.
    const int row_base = tm * BM + 64 * wm + (int)g4;
#pragma unroll
    for (int mi = 0; mi < 8; ++mi) {
        const int row = row_base + 8 * mi;
        if (row >= M) continue;
        double *crow = C + (int64_t)row * ldc;
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const int col = tn * BN + 32 * wn + 16 * q + 4 * (int)p;
            const double v0 = acc[mi][2 * q][0], v1 = acc[mi][2 * q + 1][0];
            const double v2 = acc[mi][2 * q][1], v3 = acc[mi][2 * q + 1][1];
            if (elem_mask) {   // recompute set: only the flagged elements (4 bits of one word)
                const uint32_t bits = col < N ? elem_mask[(int64_t)row * ld_emask + (col >> 5)] >> (col & 31) : 0u;
                if ((bits & 1u) && col < N) crow[col] = v0;
                if ((bits & 2u) && col + 1 < N) crow[col + 1] = v1;
                if ((bits & 4u) && col + 2 < N) crow[col + 2] = v2;
                if ((bits & 8u) && col + 3 < N) crow[col + 3] = v3;
            } else if (vec_ok && col + 3 < N) {
                *reinterpret_cast<double2 *>(crow + col) = make_double2(v0, v1);
                *reinterpret_cast<double2 *>(crow + col + 2) = make_double2(v2, v3);
            } else {
                if (col < N) crow[col] = v0;
                if (col + 1 < N) crow[col + 1] = v1;
                if (col + 2 < N) crow[col + 2] = v2;
                if (col + 3 < N) crow[col + 3] = v3;
            }
        }
    }
}

static bool make_map_2d(EncodeTiledFn enc, CUtensorMap *m, CUtensorMapDataType dt, int elem, const void *ptr,
                        uint64_t inner, uint64_t outer, uint64_t ld_elems, uint32_t box_inner, uint32_t box_outer,
                        CUtensorMapSwizzle swz) {
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {ld_elems * (uint64_t)elem};
    cuuint32_t box[2] = {box_inner, box_outer};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(m, dt, 2, const_cast<void *>(ptr), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// CTA rows for a grid of M x N, from a wave model with W = the time of one
// 128 x 128 tile on an SM: 128-row grid ceil(t128 / sms) W; 64-row grid
// W / (2 K1_E1) when every CTA has an SM to itself, else ceil(t64 / 2 sms)
// waves of two co-resident CTAs at K1_E2 of the 128-row rate.  Constants from
// tools/k1_shape_sweep.py on the B200 (profiles/r01_k1_shape_sweep.jsonl).
// DYNAMIC keeps 128 x 128 tiles: every Worker claims from one tile grid.
static int k1_pick_bm(int64_t M, int64_t N, int sms, bool dynamic) {
    const char *f = getenv("PDL_K1_BM");   // measurement knob: force 64 or 128
    if (f && (atoi(f) == 64 || atoi(f) == 128)) return atoi(f);
    if (dynamic || sms <= 0) return 128;
    const int64_t tn = (N + 127) / 128;
    const int64_t t128 = (M + 127) / 128 * tn, t64 = (M + 63) / 64 * tn;
    const double w128 = (double)((t128 + sms - 1) / sms);
    const double w64 =
        t64 <= sms ? 0.5 / K1_E1 : (double)((t64 + 2 * sms - 1) / (2 * sms)) / K1_E2;
    return w64 < w128 ? 64 : 128;
}

template <int BM_>
static cudaError_t launch_k1_shape(EncodeTiledFn enc, const double *A, int64_t lda, const double *B, int64_t ldb,
                                   double *C, int64_t ldc, int64_t M, int64_t N, int64_t K, int dev,
                                   cudaStream_t stream, int *dyn_next, int *dyn_mine, const uint32_t *tile_mask,
                                   int64_t ld_mask, const uint32_t *elem_mask, int64_t ld_emask) {
    using S = k1::Shape<BM_>;
    CUtensorMap ta, tb;
    if (!make_map_2d(enc, &ta, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 8, A, (uint64_t)K, (uint64_t)M, (uint64_t)lda, S::BK,
                     S::BM, CU_TENSOR_MAP_SWIZZLE_128B))
        return cudaErrorInvalidValue;
    if (!make_map_2d(enc, &tb, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 8, B, (uint64_t)N, (uint64_t)K, (uint64_t)ldb, 16,
                     S::BK, CU_TENSOR_MAP_SWIZZLE_128B))
        return cudaErrorInvalidValue;
    static bool attr_done[64] = {false};
    if (dev < 64 && !attr_done[dev]) {
        cudaError_t e =
            cudaFuncSetAttribute(dgemm_k1_kernel<BM_>, cudaFuncAttributeMaxDynamicSharedMemorySize, S::SMEM_BYTES);
        if (e != cudaSuccess) return e;
        attr_done[dev] = true;
    }
    const int tiles_m = (int)((M + S::BM - 1) / S::BM), tiles_n = (int)((N + S::BN - 1) / S::BN);
    const int vec_ok = ((reinterpret_cast<uintptr_t>(C) & 15u) == 0 && (ldc & 1) == 0) ? 1 : 0;
    const char *gm = getenv("PDL_GROUP_M_K1");   // raster tuning knob
    const int group_m = gm && atoi(gm) > 0 ? atoi(gm) : k1::GROUP_M * (128 / BM_);
    dgemm_k1_kernel<BM_><<<tiles_m * tiles_n, S::THREADS, S::SMEM_BYTES, stream>>>(
        ta, tb, C, ldc, (int)M, (int)N, (int)K, tiles_m, tiles_n, group_m, vec_ok, dyn_next, dyn_mine, tile_mask,
        ld_mask, elem_mask, ld_emask);
    return cudaGetLastError();
}

static int g_worker_sms = 0;
void set_worker_sms(int sms) { g_worker_sms = sms > 0 ? sms : 0; }
int worker_sms() {
    if (g_worker_sms > 0) return g_worker_sms;
    int dev = 0;
    cudaGetDevice(&dev);
    static int sm_count[64] = {0};
    if (dev < 64 && !sm_count[dev]) cudaDeviceGetAttribute(&sm_count[dev], cudaDevAttrMultiProcessorCount, dev);
    return dev < 64 ? sm_count[dev] : 148;
}

// Host launcher.  A: rows x K (lda), B: K x cols (ldb), both device-resident,
// 16 B aligned base, lda*8 and ldb*8 multiples of 16 (checked by the runtime).
cudaError_t launch_dgemm_k1(EncodeTiledFn enc, const double *A, int64_t lda, const double *B, int64_t ldb,
                            double *C, int64_t ldc, int64_t M, int64_t N, int64_t K, cudaStream_t stream,
                            int *dyn_next, int *dyn_mine, const uint32_t *tile_mask, int64_t ld_mask,
                            const uint32_t *elem_mask, int64_t ld_emask) {
    if (M <= 0 || N <= 0) return cudaSuccess;
    int dev = 0;
    cudaGetDevice(&dev);
    const int sms = worker_sms();
    if (k1_pick_bm(M, N, sms, dyn_next != nullptr) == 64)
        return launch_k1_shape<64>(enc, A, lda, B, ldb, C, ldc, M, N, K, dev, stream, dyn_next, dyn_mine, tile_mask,
                                   ld_mask, elem_mask, ld_emask);
    return launch_k1_shape<128>(enc, A, lda, B, ldb, C, ldc, M, N, K, dev, stream, dyn_next, dyn_mine, tile_mask,
                                ld_mask, elem_mask, ld_emask);
}


}  // namespace pdlk
