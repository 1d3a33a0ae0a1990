// kernels.h -- internal interface between the runtime (pdl_runtime.cu) and
// the sm_100a tile kernels.  Not part of the public C ABI.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

namespace pdlk {

// cuTensorMapEncodeTiled, fetched through cudaGetDriverEntryPoint so the
// library never links libcuda directly (it must load on GPU-less hosts).
typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// K1 -- FP64 DMMA tile kernel.  Requirements (checked by the caller):
// A, B device pointers, 16 B aligned, lda*8 % 16 == 0, ldb*8 % 16 == 0.
cudaError_t launch_dgemm_k1(EncodeTiledFn enc, const double *A, int64_t lda, const double *B, int64_t ldb,
                            double *C, int64_t ldc, int64_t M, int64_t N, int64_t K, cudaStream_t stream);
int k1_smem_bytes();

// K3 -- TF32 hi/lo split pre-pass.  Kp = K rounded up to K2's BK (32).
//  split_rows:   A (M x K, lda, fp32)  -> Ahi, Alo  (M x Kp, K-major, zero padded)
//  split_cols_t: B (K x N, ldb, fp32)  -> Bhi, Blo  (N x Kp, K-major = B^T, zero padded)
constexpr int K2_BK = 32;
cudaError_t launch_split_rows(const float *A, int64_t lda, int64_t M, int64_t K, float *hi, float *lo, int64_t Kp,
                              cudaStream_t s);
cudaError_t launch_split_cols_t(const float *B, int64_t ldb, int64_t K, int64_t N, float *hi, float *lo, int64_t Kp,
                                cudaStream_t s);

// K2 -- 3xTF32 tcgen05 GEMM on the split operands:
//  C (M x N, ldc, fp32) = Ahi*Bhi^T + Ahi*Blo^T + Alo*Bhi^T   (hi/lo: M x Kp / N x Kp)
cudaError_t launch_gemm_3xtf32(EncodeTiledFn enc, const float *Ahi, const float *Alo, const float *Bhi,
                               const float *Blo, int64_t Kp, float *C, int64_t ldc, int64_t M, int64_t N,
                               cudaStream_t stream);
// K2 v3 -- same contract on a CTA pair (tcgen05 cta_group::2, 256 x 256 tiles).
cudaError_t launch_gemm_3xtf32_2sm(EncodeTiledFn enc, const float *Ahi, const float *Alo, const float *Bhi,
                                   const float *Blo, int64_t Kp, float *C, int64_t ldc, int64_t M, int64_t N,
                                   cudaStream_t stream);

}  // namespace pdlk
