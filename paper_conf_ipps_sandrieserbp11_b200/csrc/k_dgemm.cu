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
//  * Bank-conflict-free fragment loads: within each 16-wide K block the four
//    k4 MMA steps take k = {0,1,4,5}, {2,3,6,7}, {8,9,12,13}, {10,11,14,15}
//    (same permutation for A and B), which with the 128B swizzle makes every
//    64-bit fragment load exactly 2 shared-memory wavefronts.  The summation
//    order per C element is fixed by this kernel alone, so results do not
//    depend on the Worker rectangle or task tile (bitwise invariance, pin P7).
//  * CTA tile 128 x 128, grouped rasterisation for L2 reuse, masked
//    vectorised (16 B) epilogue straight from the accumulators.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"
#include "ptx.cuh"

namespace pdlk {

namespace k1 {
constexpr int BM = 128, BN = 128, BK = 16, STAGES = 4;
constexpr int A_BYTES = BM * BK * 8;   // 16 KiB
constexpr int B_BYTES = BK * BN * 8;   // 16 KiB, as BN/16 sub-boxes of 16 x 16 doubles
constexpr int B_SUB_BYTES = BK * 16 * 8;
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int NCONS = 8;               // DMMA warps; thread 0 also issues the TMA loads
constexpr int THREADS = NCONS * 32;    // 256: keeps the 255-register budget per thread
constexpr int GROUP_M = 16;            // tile rows per raster group
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 2 * STAGES * 8 + 1024;
}  // namespace k1

// 128B-swizzled byte offset of (row, 8-byte column j in [0,16)) inside a
// buffer of 128-byte rows whose base is 1024-byte aligned.
__device__ __forceinline__ uint32_t swz128(uint32_t row, uint32_t j) {
    return row * 128u + ((((j >> 1) ^ (row & 7u)) << 4) | ((j & 1u) << 3));
}

__device__ __forceinline__ double lds64(uint32_t addr) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(addr));
    return v;
}

__device__ __forceinline__ void dmma(double &c0, double &c1, double a, double b) {
    asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

__global__ void __launch_bounds__(k1::THREADS, 1)
    dgemm_k1_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                    double *__restrict__ C, int64_t ldc, int M, int N, int K, int tiles_m, int tiles_n,
                    int vec_ok) {
    using namespace k1;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t base = (smem_u32(smem_raw) + 1023u) & ~1023u;
    const uint32_t bar_full = base + STAGES * STAGE_BYTES;
    const uint32_t bar_empty = bar_full + STAGES * 8;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    // grouped raster: GROUP_M tile rows sweep the tile columns together
    const int bid = blockIdx.x;
    const int per_group = GROUP_M * tiles_n;
    const int g = bid / per_group;
    const int first_m = g * GROUP_M;
    const int gsz = min(tiles_m - first_m, GROUP_M);
    const int tm = first_m + (bid % per_group) % gsz;
    const int tn = (bid % per_group) / gsz;

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
    const int wm = warp >> 2, wn = warp & 3;   // 2 x 4 warps, warp tile 64 x 32
    const uint32_t g4 = (uint32_t)lane >> 2;   // groupID
    const uint32_t p = (uint32_t)lane & 3u;    // thread in group -> MMA k index
    const uint32_t kperm = (p & 1u) + ((p >> 1) << 2);   // {0,1,4,5}

    double acc[8][4][2];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;

    // per-lane constant parts of the fragment addresses
    const uint32_t arow0 = 64u * wm + g4;              // + 8*mi
    const uint32_t bcol0 = 32u * wn + g4;              // + 8*ni  (column inside the CTA tile)

    for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % STAGES;
        const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
        mbar_wait(bar_full + 8 * s, ph);
        const uint32_t sa = base + s * STAGE_BYTES;
        const uint32_t sb = sa + A_BYTES;
#pragma unroll
        for (int step = 0; step < 4; ++step) {
            const uint32_t k = (uint32_t)((step & 1) * 2 + (step >> 1) * 8) + kperm;
            double a[8], b[4];
#pragma unroll
            for (int mi = 0; mi < 8; ++mi) a[mi] = lds64(sa + swz128(arow0 + 8u * mi, k));
#pragma unroll
            for (int ni = 0; ni < 4; ++ni) {
                const uint32_t n = bcol0 + 8u * ni;
                b[ni] = lds64(sb + (n >> 4) * B_SUB_BYTES + swz128(k, n & 15u));
            }
#pragma unroll
            for (int mi = 0; mi < 8; ++mi)
#pragma unroll
                for (int ni = 0; ni < 4; ++ni) dmma(acc[mi][ni][0], acc[mi][ni][1], a[mi], b[ni]);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(bar_empty + 8 * s);
        if (threadIdx.x == 0 && kb + STAGES < nk) {
            mbar_wait(bar_empty + 8 * s, ph);
            issue(kb + STAGES);
        }
    }

    // ---------------- epilogue: registers -> global (masked, 16 B when aligned) ----------------
    const int row_base = tm * BM + 64 * wm + (int)g4;
    const int col_base = tn * BN + 32 * wn + 2 * (int)p;
#pragma unroll
    for (int mi = 0; mi < 8; ++mi) {
        const int row = row_base + 8 * mi;
        if (row >= M) continue;
        double *crow = C + (int64_t)row * ldc;
#pragma unroll
        for (int ni = 0; ni < 4; ++ni) {
            const int col = col_base + 8 * ni;
            if (vec_ok && col + 1 < N) {
                *reinterpret_cast<double2 *>(crow + col) = make_double2(acc[mi][ni][0], acc[mi][ni][1]);
            } else {
                if (col < N) crow[col] = acc[mi][ni][0];
                if (col + 1 < N) crow[col + 1] = acc[mi][ni][1];
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

int k1_smem_bytes() { return k1::SMEM_BYTES; }

// Host launcher.  A: rows x K (lda), B: K x cols (ldb), both device-resident,
// 16 B aligned base, lda*8 and ldb*8 multiples of 16 (checked by the runtime).
cudaError_t launch_dgemm_k1(EncodeTiledFn enc, const double *A, int64_t lda, const double *B, int64_t ldb,
                            double *C, int64_t ldc, int64_t M, int64_t N, int64_t K, cudaStream_t stream) {
    using namespace k1;
    if (M <= 0 || N <= 0) return cudaSuccess;
    CUtensorMap ta, tb;
    if (!make_map_2d(enc, &ta, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 8, A, (uint64_t)K, (uint64_t)M, (uint64_t)lda, BK, BM,
                     CU_TENSOR_MAP_SWIZZLE_128B))
        return cudaErrorInvalidValue;
    if (!make_map_2d(enc, &tb, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 8, B, (uint64_t)N, (uint64_t)K, (uint64_t)ldb, 16, BK,
                     CU_TENSOR_MAP_SWIZZLE_128B))
        return cudaErrorInvalidValue;
    int dev = 0;
    cudaGetDevice(&dev);
    static bool attr_done[64] = {false};
    if (dev < 64 && !attr_done[dev]) {
        cudaError_t e = cudaFuncSetAttribute(dgemm_k1_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
        if (e != cudaSuccess) return e;
        attr_done[dev] = true;
    }
    const int tiles_m = (int)((M + BM - 1) / BM), tiles_n = (int)((N + BN - 1) / BN);
    const int vec_ok = ((reinterpret_cast<uintptr_t>(C) & 15u) == 0 && (ldc & 1) == 0) ? 1 : 0;
    dgemm_k1_kernel<<<tiles_m * tiles_n, THREADS, SMEM_BYTES, stream>>>(ta, tb, C, ldc, (int)M, (int)N, (int)K,
                                                                        tiles_m, tiles_n, vec_ok);
    return cudaGetLastError();
}

}  // namespace pdlk
