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

// SM count of the Worker whose kernels launch next: its green-context partition
// (PDL property SM_LIMIT) or 0 for the whole device.  The runtime sets it before
// a Worker's launches (one Master thread drives the library); the shape pickers
// and persistent grids size their wave models by worker_sms().
void set_worker_sms(int sms);
int worker_sms();   // the partition's SMs if set, else the current device's

// K1 -- FP64 DMMA tile kernel.  Requirements (checked by the caller):
// A, B device pointers, 16 B aligned, lda*8 % 16 == 0, ldb*8 % 16 == 0.
cudaError_t launch_dgemm_k1(EncodeTiledFn enc, const double *A, int64_t lda, const double *B, int64_t ldb,
                            double *C, int64_t ldc, int64_t M, int64_t N, int64_t K, cudaStream_t stream,
                            int *dyn_next = nullptr, int *dyn_mine = nullptr, const uint32_t *tile_mask = nullptr,
                            int64_t ld_mask = 0, const uint32_t *elem_mask = nullptr, int64_t ld_emask = 0);
// dyn_next / dyn_mine (K1, K2): DYNAMIC distribution -- CTAs claim raster tiles
// from the shared counter *dyn_next and count their claims in *dyn_mine.
// tile_mask (K1): compute only the 128 x 128 tiles t with tile_mask[(row / 128) *
// ld_mask + col / 128] != 0; the other CTAs exit before touching memory.
// elem_mask: of those, store only the elements whose bit (col % 32) of
// elem_mask[row * ld_emask + col / 32] is set (the Ozaki-II certificate's recompute
// set).  A stored element is bitwise the plain K1 result.

// K3 -- TF32 hi/lo split pre-pass.  Kp = K rounded up to K2's BK (32).
//  split_rows:   A (M x K, lda, fp32)  -> Ahi, Alo  (M x Kp, K-major, zero padded; row stride
//                ldo floats, default Kp -- the packed prepared-A rows [hi | lo] use 2 Kp)
//  split_cols_t: B (K x N, ldb, fp32)  -> Bhi, Blo  (N x Kp, K-major = B^T, zero padded)
constexpr int K2_BK = 32;
// mix = 1 (FP32 task variant "tf32bf16", R22): hi as above; the `lo` plane
//                holds bf16 pairs per 32-wide K block b -- halves [64 b, 64 b + 32) =
//                rn_bf16(hi), [64 b + 32, 64 b + 64) = rn_bf16(x - hi) (same bytes per row).
cudaError_t launch_split_rows(const float *A, int64_t lda, int64_t M, int64_t K, float *hi, float *lo, int64_t Kp,
                              cudaStream_t s, int64_t ldo = 0, int mix = 0);
cudaError_t launch_split_cols_t(const float *B, int64_t ldb, int64_t K, int64_t N, float *hi, float *lo, int64_t Kp,
                                cudaStream_t s, int mix = 0);

// K2 -- 3xTF32 tcgen05 GEMM on the split operands:
//  C (M x N, ldc, fp32) = Ahi*Bhi^T + Ahi*Blo^T + Alo*Bhi^T   (hi/lo: M x Kp / N x Kp;
//  lda_s = row stride of Ahi / Alo in floats, 0 = Kp)
// mix = 1 (R22): the lo planes are the bf16 [hi' | lo'] planes of the mixed split and
//  C = Ahi*Bhi^T (kind::tf32) + Ahi'*Blo'^T + Alo'*Bhi'^T (kind::f16, BF16 operands):
//  two TF32-equivalent tensor passes per K block instead of three.
cudaError_t launch_gemm_3xtf32(EncodeTiledFn enc, const float *Ahi, const float *Alo, const float *Bhi,
                               const float *Blo, int64_t Kp, float *C, int64_t ldc, int64_t M, int64_t N,
                               cudaStream_t stream, int64_t lda_s = 0, int mix = 0);
// K6/K7 -- FP64 DGEMM variant "ozaki2" (Ozaki scheme II: integer scaling and the
// Chinese remainder theorem over INT8 GEMMs, k_ozaki2.cu).  A' = rint(A 2^(p-e_i))
// row-wise, B' = rint(B 2^(p-f_j)) column-wise (|A'|, |B'| <= 2^p); for each of n
// pairwise-coprime moduli m_t <= 256 one INT8 GEMM of the residues (exact INT32)
// reduced mod m_t into a byte plane; X = A'B' is rebuilt from the n planes by CRT
// (exact: |X| < M/2, M = prod m_t) and C = X 2^(e_i + f_j - 2p).
// Residues: A8 = rows x ld8, row layout [chunk][modulus][Kc]; Bt8 = cols x ld8 the
// same for B^T.  Planes: R + (c n + t) * plane, rows x ldr bytes each.
constexpr int OZ2_MAX_MODULI = 14;        // sum_t u_t W_t < 2^128 (u_t < 256, W_t < M < 2^111)
constexpr int64_t OZ2_KC_MAX = 65536;     // |sum r_a r_b| <= Kc 2^14 < 2^31
struct Ozaki2Plan {
    int n = 0;                            // moduli in use
    int p = 0;                            // integer scaling bits
    int nch = 1;
    int check = 0;                        // 1: plane n of the operands is the certificate operand
    int np = 0;                           // operand planes per K chunk: n + check
    int64_t Kc = 0, ld8 = 0;
    size_t a8_bytes = 0, b8_bytes = 0;
    int m[OZ2_MAX_MODULI] = {};
    unsigned long long W[OZ2_MAX_MODULI][2] = {};   // CRT weights (lo, hi words)
    unsigned long long Mw[2] = {}, Hw[2] = {};      // M and floor(M / 2)
    double Md = 0.0;
};
// nmod = 0: the fewest moduli that give p >= bits for this K chunk.  guard: add the
// certificate plane when the plan admits it (oz2_guard_ok).
Ozaki2Plan ozaki2_plan(int64_t rows, int64_t cols, int64_t K, int nmod, int bits, bool guard = false);
// The componentwise certificate (R21) needs one K chunk, an exact INT32
// certificate sum (127^2 Kc < 2^31) and the u64 row / column sums ((2^(p+1)+1) K < 2^63).
bool oz2_guard_ok(const Ozaki2Plan &P, int64_t K);
// Certificate of one Ozaki-II launch (R21).  With A' = rint(A 2^(p-e_i))
// and B' = rint(B 2^(p-f_j)) the componentwise error of C_ij is at most
//   2^(e_i+f_j-2p-2) (sa_i + sb_j + min(sa_i, sb_j))  + rounding of X to double,
// sa_i = sum_k (2|A'_ik| + 1)[A_ik != 0] (sb_j likewise), and D_ij = sum_k |A_ik||B_kj|
// is at least 2^(e_i+f_j-14) X^c_ij, X^c = a^c b^c with a^c_ik = max(0, |A'_ik| - 1) >>
// (p - 7) in [0, 127] (b^c likewise): the certificate plane, one more INT8 GEMM.  A
// 128 x 128 tile holding an element whose bound exceeds tau D_ij is flagged and
// recomputed by K1 (IEEE FP64); K1 stores only the flagged elements, so every
// element's value depends on its own certificate alone (bitwise invariance, R14).
struct Oz2Guard {
    unsigned long long *sa = nullptr;     // rows of the launch's rectangle (stride sa_ld)
    int64_t sa_ld = 1;
    unsigned long long *sb = nullptr;     // its columns
    double *sbd = nullptr;                // cols doubles of scratch (the epilogue's column term)
    uint32_t *flags = nullptr;            // tile (row / 128, col / 128) at flags[(row / 128) * ldf + col / 128]
    int64_t ldf = 0;
    uint32_t *emask = nullptr;            // element (row, col): bit col % 32 of emask[row * ldw + col / 32]
    int64_t ldw = 0;
    unsigned *fallback = nullptr;         // [0] += flagged tiles, [1] += flagged elements (stats)
    double tau = 5e-13;
    // Sign-uniform rows and columns (R23; rsign null = off).  Where row i and
    // column j each hold entries of one sign, D_ij = |C_ij| and the CRT pass certifies the
    // element against its own |X|; the certificate GEMM checks the other elements and is
    // skipped when no row or column of the launch mixes signs (*sign_word == 0 after the
    // scan in its column-term pass).  Sign bits: bit 0 = a positive entry, bit 1 = a
    // negative one.
    const unsigned *rsign = nullptr;      // rows of the launch, stride rsign_ld (the packed row's pad word)
    int64_t rsign_ld = 1;
    const unsigned *csign = nullptr;      // columns of the launch
    unsigned *sign_word = nullptr;        // the launch's "some row or column mixes signs" word
    double *sbu = nullptr;                // per column (written by the column-term pass): sb_j rounded
                                          // up to double, -1 for a column that mixes signs
    unsigned long long *sbmax = nullptr;  // the launch's largest uniform column term (double bits)
    double *rowT = nullptr;               // per row of the launch: the CRT pass's bound T_i (0: none)
};
// thr4 = 4 (tau / (1 + tau) - 2^-52), rounded down: the R23 certificate's scale
inline double oz2_uniform_thr4(double tau) { return 4.0 * (tau / (1.0 + tau) - 0x1p-52) * (1.0 - 0x1p-48); }
// Persistent K6 launches per K chunk for n moduli on a rows x cols rectangle with
// `clusters` co-resident CTA pairs (k_ozaki.cu).
int oz2_launches_per_chunk(int n, int64_t rows, int64_t cols, int clusters);
// sa / sb (P.check): the certificate's row / column sums, zeroed and accumulated here.
// lda8: row stride of A8 in bytes (0 = P.ld8); ea_ld / sa_ld: strides of ea / sa in
// elements -- the packed prepared-A rows below use lda8 = P.ld8 + 16, ea_ld = lda8 / 4,
// sa_ld = lda8 / 8.
// rsign (optional, stride ea_ld): each row's sign bits (R23) -- the pad word after e_i
// in the packed prepared rows, so they travel with exchanged rows.
cudaError_t launch_ozaki2_split_a(const double *A, int64_t lda, int64_t rows, int64_t K, const Ozaki2Plan &P,
                                  int8_t *A8, int *ea, cudaStream_t s, int *launches = nullptr,
                                  unsigned long long *sa = nullptr, int64_t lda8 = 0, int64_t ea_ld = 1,
                                  int64_t sa_ld = 1, unsigned *rsign = nullptr);
// Prepared A rows of the ozaki2 variant (what PDL_TASK_PREP_A writes and
// PDL_TASK_PREPARED_A reads): [residues: P.ld8 bytes][e_i: int32][sign bits: u32][sa_i: u64].
inline int64_t oz2_prep_row_bytes(const Ozaki2Plan &P) { return P.ld8 + 16; }
// csign (optional): per column sign bits (bit 0 positive, bit 1 negative entry; R23).
cudaError_t launch_ozaki2_split_b(const double *B, int64_t ldb, int64_t K, int64_t cols, const Ozaki2Plan &P,
                                  int8_t *Bt8, int *fb, unsigned long long *bmax, cudaStream_t s,
                                  unsigned long long *sb = nullptr, unsigned *csign = nullptr);
// guard (P.check): the certificate GEMM runs as one more item of the persistent
// launches and flags tiles into guard->flags (zeroed by the caller).
cudaError_t launch_ozaki2_gemm(EncodeTiledFn enc, const int8_t *A8, const int8_t *Bt8, const Ozaki2Plan &P,
                               uint8_t *R, int64_t ldr, int64_t plane, int64_t rows, int64_t cols, cudaStream_t s,
                               int *launches, const Oz2Guard *guard = nullptr, int64_t lda8 = 0);
// The plan admits the FP64-pipe CRT pass (M < 2^117, M >= 2^(2p + lk + 1) (1 + 1/64));
// otherwise launch_ozaki2_reconstruct uses the 128-bit integer pass.  PDL_OZ2_CRT=int
// forces the integer pass.
bool oz2_crt_fast_ok(const Ozaki2Plan &P);
// guard with rsign (R23): the FP64-pipe CRT pass certifies the elements of sign-uniform
// rows and columns against |X| (D = |C| there) and flags the failing ones for K1.
cudaError_t launch_ozaki2_reconstruct(const uint8_t *R, int64_t ldr, int64_t plane, const int *ea, const int *fb,
                                      const Ozaki2Plan &P, double *C, int64_t ldc, int64_t rows, int64_t cols,
                                      cudaStream_t s, int64_t ea_ld = 1, const Oz2Guard *guard = nullptr);

// K2 v3 -- same contract on a CTA pair (tcgen05 cta_group::2, 256 x 256 tiles).
cudaError_t launch_gemm_3xtf32_2sm(EncodeTiledFn enc, const float *Ahi, const float *Alo, const float *Bhi,
                                   const float *Blo, int64_t Kp, float *C, int64_t ldc, int64_t M, int64_t N,
                                   cudaStream_t stream, int *dyn_next = nullptr, int *dyn_mine = nullptr,
                                   int64_t lda_s = 0, int mix = 0);

}  // namespace pdlk
