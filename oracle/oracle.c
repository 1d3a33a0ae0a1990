/*
 * oracle.c -- CPU oracle for the PDL-mapped blocked matrix multiply.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ipps_sandrieserbp11_b200/csrc); neither side includes the other.
 *
 * What it computes (the plain definition the method reaches up to rounding):
 *
 *     C_ij = sum_{k=0}^{K-1} A_ik * B_kj          0 <= i < M, 0 <= j < N
 *
 * PAPER.md L1402-1406 (SS IV-D "Preliminary Experiment"): "The serial input
 * program performs a double precision matrix multiplication of two
 * 8192x8192 matrices (DGEMM)".  Tasks are "self-contained units of work ...
 * with input and output parameters" sharing one signature across variants
 * (L1032-1039), so every task variant must reach this same product.
 * Readings (R1-R3): alpha = 1, beta = 0 (C is access mode `write`,
 * L1184-1186); row-major storage, leading dimension = number of columns.
 *
 * Algorithm: triple loop in i-k-j order, k ascending for
 * every element, inputs promoted exactly to double, double accumulator.
 * Besides Cref it returns D = (|A|)(|B|) accumulated in the same loop; the
 * parity tests scale the error by D (R13).
 *
 * Build: gcc -O3 -fopenmp -ffp-contract=off -shared -fPIC (no -ffast-math),
 * so the j loop vectorises without reassociation and results are bitwise
 * reproducible.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* dtype codes: 0 = float64 inputs, 1 = float32 inputs (promoted exactly). */

static void one_row(int dtype, const void *A, const void *B, int64_t i,
                    int64_t N, int64_t K, double *acc, double *mag)
{
    for (int64_t j = 0; j < N; ++j) { acc[j] = 0.0; mag[j] = 0.0; }
    for (int64_t k = 0; k < K; ++k) {
        double a;
        if (dtype == 0) a = ((const double *)A)[i * K + k];
        else            a = (double)((const float *)A)[i * K + k];
        double aa = fabs(a);
        if (dtype == 0) {
            const double *b = (const double *)B + k * N;
            for (int64_t j = 0; j < N; ++j) {
                acc[j] += a * b[j];
                mag[j] += aa * fabs(b[j]);
            }
        } else {
            const float *b = (const float *)B + k * N;
            for (int64_t j = 0; j < N; ++j) {
                double bj = (double)b[j];
                acc[j] += a * bj;
                mag[j] += aa * fabs(bj);
            }
        }
    }
}

/*
 * oracle_matmul_rows: compute rows[0..nrows) of Cref and D.
 *   A: M x K row-major, B: K x N row-major (dtype as above), host memory.
 *   rows: row indices (any order, each < M); NULL means rows 0..nrows-1.
 *   Cref, D: nrows x N doubles, row r of the output is row rows[r] of C.
 *   D may be NULL (then only Cref is produced).
 *   nthreads <= 0: OpenMP default.
 * Returns 0, or -1 on bad arguments.
 */
int oracle_matmul_rows(int dtype, const void *A, const void *B,
                       int64_t M, int64_t N, int64_t K,
                       const int64_t *rows, int64_t nrows,
                       double *Cref, double *D, int nthreads)
{
    if (dtype != 0 && dtype != 1) return -1;
    if (M < 0 || N < 0 || K < 0 || nrows < 0) return -1;
    if (nrows == 0 || N == 0) return 0;
    if (!Cref) return -1;
    if (K > 0 && (!A || !B)) return -1;
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t i = rows ? rows[r] : r;
        if (i < 0 || i >= M) return -1;
    }
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#endif
    int bad = 0;
#pragma omp parallel
    {
        double *mag_scratch = (double *)malloc((size_t)N * sizeof(double));
        if (!mag_scratch) {
#pragma omp atomic write
            bad = 1;
        }
#pragma omp for schedule(dynamic, 1)
        for (int64_t r = 0; r < nrows; ++r) {
            if (!mag_scratch) continue;
            int64_t i = rows ? rows[r] : r;
            double *mag = D ? D + r * N : mag_scratch;
            one_row(dtype, A, B, i, N, K, Cref + r * N, mag);
        }
        free(mag_scratch);
    }
    return bad ? -1 : 0;
}

/* Full product: rows 0..M-1. */
int oracle_matmul(int dtype, const void *A, const void *B,
                  int64_t M, int64_t N, int64_t K,
                  double *Cref, double *D, int nthreads)
{
    return oracle_matmul_rows(dtype, A, B, M, N, K, NULL, M, Cref, D, nthreads);
}

/* Number of threads OpenMP will use (for the bench's `cores` field). */
int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
