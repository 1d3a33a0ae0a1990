// k_ozaki2.cu -- K6/K7: the FP64 DGEMM task variant "ozaki2" on the INT8 tensor
// cores (Ozaki scheme II: integer scaling + Chinese remainder theorem),
// SURVEY.md SS8(f) NEXT-1, a third implementation variant of the DGEMM task
// (task repository / static pre-selection, PAPER.md L1033-1039, L1307-1326;
// PDL property DGEMM_VARIANT = "ozaki2").
//
// Method (Ozaki, Uchino, Imamura 2025, "Ozaki scheme II"; K6):
//   scaling   A'_ik = rint(A_ik 2^{p-e_i}),  B'_kj = rint(B_kj 2^{p-f_j})   (|.| <= 2^p)
//             e_i: max_k |A_ik| < 2^{e_i};  f_j likewise for columns of B
//   residues  for pairwise-coprime m_t <= 256: a_t = A' mod m_t in [-128, 127]
//   GEMMs     X_t = sum_k a_t b_t  (exact INT32 on tcgen05 kind::i8), u_t = X_t mod m_t
//   CRT       X = A'B' is the unique integer in (-M/2, M/2] with X = u_t (mod m_t),
//             M = prod m_t; exact because |X| <= K 2^{2p} < M/2 by the choice of p
//   result    C_ij = X_ij 2^{e_i + f_j - 2p}
// The only rounding is the scaling of A and B to p-bit integers (|err| <= 2^{e_i-p-1}
// per element) and the final conversion of X to double; n moduli replace the
// S(S+1)/2 slice products of scheme I (13 GEMMs instead of 21 at K = 16384 for
// p = 43).  Inputs must be finite (R15).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <algorithm>

#include "kernels.h"

namespace pdlk {

// Pairwise-coprime moduli <= 256 (2^8, 3*5*17, 11*23, 251, 13*19, primes, 7*31, ...),
// largest first: residues in [-128, 127] fit int8 and products sum exactly in INT32.
static const int kModuli[OZ2_MAX_MODULI] = {256, 255, 253, 251, 247, 241, 239, 233, 229, 227, 223, 217, 211, 199};

__constant__ double c_oz2_m[OZ2_MAX_MODULI];
__constant__ double c_oz2_inv[OZ2_MAX_MODULI];
__constant__ int c_oz2_mi[OZ2_MAX_MODULI];

// ------------------------------------------------------------------------
// plan (host): moduli count, scaling bits, CRT constants
// ------------------------------------------------------------------------
typedef unsigned __int128 u128;

static int inv_mod(int a, int m) {   // a^-1 mod m (gcd(a, m) = 1)
    int t = 0, nt = 1, r = m, nr = a % m;
    while (nr) {
        const int q = r / nr;
        int x = t - q * nt;
        t = nt;
        nt = x;
        x = r - q * nr;
        r = nr;
        nr = x;
    }
    return t < 0 ? t + m : t;
}

static int ilog2_ceil(int64_t x) {
    int b = 0;
    while (((int64_t)1 << b) < x) ++b;
    return b;
}

// Largest p <= 52 with 2^(2p+1) * 2^ceil(log2 Kc) < M (so |X| <= Kc 2^(2p) < M/2).
static int bits_for(u128 M, int64_t Kc) {
    const int lk = ilog2_ceil(Kc < 1 ? 1 : Kc);
    int p = 0;
    for (int q = 1; q <= 52; ++q)
        if (2 * q + 1 + lk < 127 && ((u128)1 << (2 * q + 1 + lk)) < M) p = q;
    return p;
}

bool oz2_guard_ok(const Ozaki2Plan &P, int64_t K) {
    return P.nch == 1 && 16129 * P.Kc < ((int64_t)1 << 31) && P.p >= 7 &&
           P.p + 2 + ilog2_ceil(K < 1 ? 1 : K) <= 62;
}

Ozaki2Plan ozaki2_plan(int64_t rows, int64_t cols, int64_t K, int nmod, int bits, bool guard) {
    Ozaki2Plan P;
    P.nch = (int)((K + OZ2_KC_MAX - 1) / OZ2_KC_MAX);
    if (P.nch < 1) P.nch = 1;
    const int64_t per = (K + P.nch - 1) / P.nch;
    P.Kc = ((per + 127) / 128) * 128;   // whole 128-byte K blocks (BK of the INT8 GEMM)
    if (P.Kc < 128) P.Kc = 128;
    int n = nmod > 0 ? (nmod > OZ2_MAX_MODULI ? OZ2_MAX_MODULI : (nmod < 2 ? 2 : nmod)) : 0;
    if (n == 0) {   // fewest moduli reaching the requested scaling bits
        u128 M = 1;
        for (n = 1; n <= OZ2_MAX_MODULI; ++n) {
            M *= (u128)kModuli[n - 1];
            if (bits_for(M, P.Kc) >= bits) break;
        }
        if (n > OZ2_MAX_MODULI) n = OZ2_MAX_MODULI;
    }
    P.n = n;
    u128 M = 1;
    for (int t = 0; t < n; ++t) {
        P.m[t] = kModuli[t];
        M *= (u128)kModuli[t];
    }
    P.p = bits_for(M, P.Kc);
    for (int t = 0; t < n; ++t) {
        const u128 Mt = M / (u128)P.m[t];
        const int r = (int)(Mt % (u128)P.m[t]);
        const u128 W = (Mt * (u128)inv_mod(r, P.m[t])) % M;
        P.W[t][0] = (unsigned long long)W;
        P.W[t][1] = (unsigned long long)(W >> 64);
    }
    P.Mw[0] = (unsigned long long)M;
    P.Mw[1] = (unsigned long long)(M >> 64);
    const u128 H = M / 2;
    P.Hw[0] = (unsigned long long)H;
    P.Hw[1] = (unsigned long long)(H >> 64);
    P.Md = (double)P.Mw[1] * 18446744073709551616.0 + (double)P.Mw[0];
    P.check = guard && oz2_guard_ok(P, K) ? 1 : 0;
    P.np = n + P.check;
    P.ld8 = (int64_t)P.nch * P.np * P.Kc;
    P.a8_bytes = (size_t)rows * P.ld8;
    P.b8_bytes = (size_t)cols * P.ld8;
    return P;
}

// ------------------------------------------------------------------------
// K7: scaling + residues (pre-pass)
// ------------------------------------------------------------------------
__device__ __forceinline__ double pow2d(int E) {   // 2^E, E in [-1022, 1023]
    return __longlong_as_double((long long)(1023 + E) << 52);
}
// x 2^E exactly as ldexp would round it (two exact-operand steps off the normal range)
__device__ __forceinline__ double scale2(double x, int E) {
    if (E >= -1022 && E <= 1023) return x * pow2d(E);
    const int E1 = E < 0 ? -1022 : 1023;
    return (x * pow2d(E1)) * pow2d(max(-1022, min(1023, E - E1)));
}
__device__ __forceinline__ int exp_of_max2(double mx) {   // mx < 2^e (0 -> 0)
    if (!(mx > 0.0)) return 0;
    int e;
    frexp(mx, &e);
    return e;
}
// v (an integer, |v| <= 2^52) mod m as a representative in [-128, 127].  Round-
// to-integer by the 1.5 * 2^52 magic constant instead of rint / F2I: t = fma(v,
// 1/m, magic) holds q = round(v/m) (one rounding of the exact product; |v/m| <
// 2^45), q = t - magic and r = v - q m are exact (|q m| < 2^53), and r + magic
// carries r in its low word -- four FP64-pipe operations, no conversion unit.
// q may be one off when v/m sits within 2^-8 of a half-integer (1/m rounded);
// the integer fix-ups fold r back into [-128, 127].
__device__ __forceinline__ int res8(double v, int t) {
    const double magic = 6755399441055744.0;   // 1.5 * 2^52
    const double m = c_oz2_m[t];
    const double q = fma(v, c_oz2_inv[t], magic) - magic;
    const double r = fma(-q, m, v);
    int ri = __double2loint(r + magic);
    const int mi = c_oz2_mi[t];
    ri -= ri > 127 ? mi : 0;
    ri += ri < -128 ? mi : 0;
    return ri;
}

// Fast residue for p <= 50 (|v| < 2^51), one DFMA and one IMAD per modulus.
// vm = v + 1.5 * 2^52 (exact), its low word = the low 32 bits of the integer v.
// q = round(v / m) is EXACT here: for odd m, v / m = n + k / m lies at least
// 1 / (2m) from a half-integer while v * rn(1/m) is within |v| / m * 2^-53 < 1 / (2m)
// of v / m; for m = 256 the reciprocal is exact.  fma(v, 1/m, magic) = q + magic
// carries q's low 32 bits in its low word, and r = v - q m (|r| <= m / 2 <= 128)
// follows exactly from the low words in wrapping 32-bit arithmetic.  r = +-128
// occurs only for m = 256, whose byte 0x80 is congruent to both.
__device__ __forceinline__ int res8_fast(double v, int vlo, int t) {
    const double qm = fma(v, c_oz2_inv[t], 6755399441055744.0);
    return vlo - __double2loint(qm) * c_oz2_mi[t];
}
// rint(x 2^sh) + 1.5 * 2^52 in one DFMA (round-to-nearest-even on the integer grid
// of [2^52, 2^53) is rint); off the normal exponent range through scale2.
__device__ __forceinline__ double scaled_magic(double x, int sh) {
    const double magic = 6755399441055744.0;
    if (sh >= -1022 && sh <= 1023) return fma(x, pow2d(sh), magic);
    return rint(scale2(x, sh)) + magic;
}

// Certificate operand of one scaled integer v = rint(x 2^(p-e)) (|v| <= 2^p):
// max(0, |v| - 1) 2^(7-p) rounded down, in [0, 127] and at most |x| 2^(7-e)
// (|v| - 1 < |x| 2^(p-e)); and the row / column sum term 2|v| + 1 for x != 0
// (|x| 2^(p-e) <= |v| + 1/2).  DESIGN.md R21.
// Both on the FP64 pipe, no conversion-unit op: x = max(|v| - 1, 0) 2^(7-p) < 2^7 is
// exact, and x + 2^52 rounded down carries floor(x) in its low word; 2|v| + 1 <
// 2^52 (p <= 50) is an exact integer whose sum with 2^52 holds it in the mantissa.
__device__ __forceinline__ int cert8(double v, int p) {
    const double x = fmax(fabs(v) - 1.0, 0.0) * pow2d(7 - p);
    return __double2loint(__dadd_rd(x, 4503599627370496.0));
}
__device__ __forceinline__ unsigned long long cert_sum(double v, bool nz, int p) {
    if (!nz) return 0ull;
    const double d = fma(2.0, fabs(v), 1.0);
    if (p <= 50) return (unsigned long long)(__double_as_longlong(d + 4503599627370496.0) - 0x4330000000000000ll);
    return (unsigned long long)d;   // < 2^53: exact
}
__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x, int width) {
    for (int o = 1; o < width; o <<= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}

// Low bytes of eight ints packed little-endian into 64 bits (PRMT, no shifts).
__device__ __forceinline__ uint64_t pack8(const int (&r)[8]) {
    const unsigned a = __byte_perm(__byte_perm(r[0], r[1], 0x0040), __byte_perm(r[2], r[3], 0x0040), 0x5410);
    const unsigned b = __byte_perm(__byte_perm(r[4], r[5], 0x0040), __byte_perm(r[6], r[7], 0x0040), 0x5410);
    return ((uint64_t)b << 32) | a;
}

// One CTA per row (grid-stride): A (rows x K) -> A8 rows [c][t][kk].
__global__ void oz2_split_rows_kernel(const double *__restrict__ A, int64_t lda, int64_t M, int64_t K, int n,
                                      int p, int64_t Kc, int nch, int8_t *__restrict__ A8, int64_t ld8,
                                      int *__restrict__ ea, int64_t ea_ld) {
    __shared__ double red[32];
    const int64_t Kpad = (int64_t)nch * Kc;
    for (int64_t i = blockIdx.x; i < M; i += gridDim.x) {
        const double *row = A + i * lda;
        double mx = 0.0;
        for (int64_t k = threadIdx.x; k < K; k += blockDim.x) mx = fmax(mx, fabs(row[k]));
        for (int o = 16; o; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = mx;
        __syncthreads();
        if (threadIdx.x < 32) {
            mx = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : 0.0;
            for (int o = 16; o; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
            if (threadIdx.x == 0) red[0] = mx;
        }
        __syncthreads();
        const int e = exp_of_max2(red[0]);
        if (threadIdx.x == 0) ea[i * ea_ld] = e;
        int8_t *out = A8 + i * ld8;
        for (int64_t k8 = (int64_t)threadIdx.x * 8; k8 < Kpad; k8 += (int64_t)blockDim.x * 8) {
            double v[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = (k8 + j < K) ? rint(scale2(row[k8 + j], p - e)) : 0.0;
            const int64_t c = k8 / Kc, kk = k8 - c * Kc;
            int8_t *o = out + (c * n) * Kc + kk;   // (no certificate plane: np == n here)
            for (int t = 0; t < n; ++t) {
                uint64_t pk = 0;
#pragma unroll
                for (int j = 0; j < 8; ++j) pk |= (uint64_t)(uint8_t)(int8_t)res8(v[j], t) << (8 * j);
                *reinterpret_cast<uint64_t *>(o + (int64_t)t * Kc) = pk;
            }
        }
        __syncthreads();
    }
}

// Two-pass A residues (the default): a row-max pass, one warp per row with
// coalesced loads, then an element-parallel residue pass over (row, 8-k group)
// items -- every thread busy and 8 independent loads in flight, instead of one CTA
// walking a row twice (oz2_split_rows_kernel, kept as PDL_OZ2_SPLIT=rows).
// rsign (R23, optional, stride ea_ld): the row's sign bits -- bit 0 a positive entry,
// bit 1 a negative one (3: the row mixes signs).
__global__ void __launch_bounds__(256) oz2_rowmax_kernel(const double *__restrict__ A, int64_t lda, int64_t M,
                                                         int64_t K, int *__restrict__ ea, int64_t ea_ld,
                                                         unsigned *__restrict__ rsign) {
    const int64_t row = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
    if (row >= M) return;
    const int lane = threadIdx.x & 31;
    const double *r = A + row * lda;
    double mx = 0.0;
    bool pos = false, neg = false;
    for (int64_t k = lane; k < K; k += 32) {
        const double v = r[k];
        mx = fmax(mx, fabs(v));
        pos |= v > 0.0;
        neg |= v < 0.0;
    }
    for (int o = 16; o; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if (lane == 0) ea[row * ea_ld] = exp_of_max2(mx);
    if (rsign) {
        pos = __any_sync(0xffffffffu, pos);
        neg = __any_sync(0xffffffffu, neg);
        if (lane == 0) rsign[row * ea_ld] = (pos ? 1u : 0u) | (neg ? 2u : 0u);
    }
}

// (256, 3): 80 registers, three CTAs per SM -- more loads in flight than the 96-register
// two-CTA build (C4: 1.57 -> 1.29 ms; a 64-register four-CTA build spills)
__global__ void __launch_bounds__(256, 3) oz2_residue_rows_kernel(const double *__restrict__ A, int64_t lda, int64_t M,
                                                               int64_t K, int n, int np, int p, int64_t Kc, int nch,
                                                               int8_t *__restrict__ A8, int64_t ld8,
                                                               const int *__restrict__ ea, int64_t ea_ld, int vec,
                                                               unsigned long long *__restrict__ sa, int64_t sa_ld) {
    const int64_t groups = (int64_t)nch * Kc / 8;   // Kc % 128 == 0
    const bool fast = p <= 50;                      // |A'| < 2^51: res8_fast (uniform)
    const bool check = np > n;                      // certificate plane n (one K chunk)
    // 2-D grid-stride: rows along y, 8-k groups along x (no 64-bit divisions)
    for (int64_t row = blockIdx.y; row < M; row += gridDim.y) {
    unsigned long long rsum = 0;
    for (int64_t g8 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g8 < groups;
         g8 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t k8 = g8 * 8;
        const double *r = A + row * lda;
        const int sh = p - ea[row * ea_ld];
        double v[8];
        if (vec && k8 + 8 <= K) {   // 16-byte aligned row and a full group: 4 x LDG.128
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const double2 x = __ldcs(reinterpret_cast<const double2 *>(r + k8) + j);
                v[2 * j] = x.x;
                v[2 * j + 1] = x.y;
            }
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = (k8 + j < K) ? r[k8 + j] : 0.0;
        }
        const int64_t c = nch == 1 ? 0 : k8 / Kc, kk = k8 - c * Kc;
        int8_t *o = A8 + row * ld8 + (c * np) * Kc + kk;
        bool nz[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) nz[j] = v[j] != 0.0;
        if (fast) {
            int lo[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const double vm = scaled_magic(v[j], sh);
                lo[j] = __double2loint(vm);
                v[j] = vm - 6755399441055744.0;
            }
            for (int t = 0; t < n; ++t) {
                int rr[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) rr[j] = res8_fast(v[j], lo[j], t);
                *reinterpret_cast<uint64_t *>(o + (int64_t)t * Kc) = pack8(rr);
            }
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = rint(scale2(v[j], sh));
            for (int t = 0; t < n; ++t) {
                int rr[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) rr[j] = res8(v[j], t);
                *reinterpret_cast<uint64_t *>(o + (int64_t)t * Kc) = pack8(rr);
            }
        }
        if (check) {
            int cc[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                cc[j] = cert8(v[j], p);
                rsum += cert_sum(v[j], nz[j], p);
            }
            *reinterpret_cast<uint64_t *>(o + (int64_t)n * Kc) = pack8(cc);
        }
    }
    if (check) {   // the warp's 32 lanes share the row (blockDim.x = 256 along k)
        rsum = warp_sum_u64(rsum, 32);
        if ((threadIdx.x & 31) == 0 && rsum) atomicAdd(sa + row * sa_ld, rsum);
    }
    }
}

// csign (R23): per column, bit 0 = a positive entry seen, bit 1 = a negative one.
__global__ void oz2_colmax_kernel(const double *__restrict__ B, int64_t ldb, int64_t K, int64_t N,
                                  unsigned long long *__restrict__ bmax, unsigned *__restrict__ csign) {
    const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (n >= N) return;
    const int64_t k0 = (int64_t)blockIdx.y * 256, k1 = min(K, k0 + 256);
    double mx = 0.0;
    unsigned sg = 0;
    for (int64_t k = k0; k < k1; ++k) {
        const double v = B[k * ldb + n];
        mx = fmax(mx, fabs(v));
        sg |= (v > 0.0 ? 1u : 0u) | (v < 0.0 ? 2u : 0u);
    }
    atomicMax(bmax + n, (unsigned long long)__double_as_longlong(mx));
    if (csign && sg) atomicOr(csign + n, sg);
}

// B (K x N) -> Bt8 (N rows of [c][t][kk]) through a shared tile stored transposed
// (32 n rows x 64 k, row pitch 66 doubles): coalesced loads along n, then each
// thread reads its column's 8 consecutive k as four 16-byte shared loads (every
// quarter-warp on distinct banks) and writes one 8-byte word per modulus.  A CTA
// walks the k tiles blockIdx.y, blockIdx.y + gridDim.y, ... of its 32 columns (one
// tile per CTA below 65536 tiles) and adds its certificate column sums with one
// atomic per column.
__global__ void __launch_bounds__(256, 3) oz2_split_cols_t_kernel(
    const double *__restrict__ B, int64_t ldb, int64_t K, int64_t N, int n, int np, int p, int64_t Kc, int nch,
    const unsigned long long *__restrict__ bmax, int8_t *__restrict__ Bt8, int64_t ld8, int *__restrict__ fb,
    unsigned long long *__restrict__ sb) {
    constexpr int PITCH = 66;
    __shared__ __align__(16) double tl[32 * PITCH];
    const int64_t n0 = (int64_t)blockIdx.x * 32;
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const int64_t Kpad = (int64_t)nch * Kc, nkt = (Kpad + 63) / 64;
    const int nl = threadIdx.x >> 3, g = threadIdx.x & 7;
    const int64_t col = n0 + nl;
    const bool check = np > n;
    const int f = col < N ? exp_of_max2(__longlong_as_double((long long)bmax[col])) : 0;
    if (blockIdx.y == 0 && g == 0 && col < N) fb[col] = f;
    unsigned long long csum = 0;
    for (int64_t kt = blockIdx.y; kt < nkt; kt += gridDim.y) {
        const int64_t k0 = kt * 64;
        __syncthreads();   // the previous tile's shared reads are done
#pragma unroll
        for (int r = ty; r < 64; r += 8) {
            const int64_t k = k0 + r, nn = n0 + tx;
            tl[tx * PITCH + r] = (k < K && nn < N) ? __ldcs(B + k * ldb + nn) : 0.0;
        }
        __syncthreads();
        const int64_t k8 = k0 + 8 * g;
        if (col >= N || k8 >= Kpad) continue;
        double v[8];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const double2 x = *reinterpret_cast<const double2 *>(&tl[nl * PITCH + 8 * g + 2 * j]);
            v[2 * j] = x.x;
            v[2 * j + 1] = x.y;
        }
        bool nz[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) nz[j] = v[j] != 0.0;
        const int64_t c = k8 / Kc, kk = k8 - c * Kc;
        int8_t *o = Bt8 + col * ld8 + (c * np) * Kc + kk;
        if (p <= 50) {
            int lo[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const double vm = scaled_magic(v[j], p - f);
                lo[j] = __double2loint(vm);
                v[j] = vm - 6755399441055744.0;
            }
            for (int t = 0; t < n; ++t) {
                int rr[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) rr[j] = res8_fast(v[j], lo[j], t);
                *reinterpret_cast<uint64_t *>(o + (int64_t)t * Kc) = pack8(rr);
            }
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = rint(scale2(v[j], p - f));
            for (int t = 0; t < n; ++t) {
                int rr[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) rr[j] = res8(v[j], t);
                *reinterpret_cast<uint64_t *>(o + (int64_t)t * Kc) = pack8(rr);
            }
        }
        if (check) {
            int cc[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                cc[j] = cert8(v[j], p);
                csum += cert_sum(v[j], nz[j], p);
            }
            *reinterpret_cast<uint64_t *>(o + (int64_t)n * Kc) = pack8(cc);
        }
    }
    if (check) {   // the 8 lanes of a column are consecutive: reduce, one atomic per column and CTA
        csum = warp_sum_u64(csum, 8);
        if (g == 0 && csum && col < N) atomicAdd(sb + col, csum);
    }
}

// ------------------------------------------------------------------------
// K6 epilogue pass: CRT reconstruction of X from the residue planes
// ------------------------------------------------------------------------
struct Oz2Crt {
    int n, nch, p;
    unsigned int W[OZ2_MAX_MODULI][4];   // CRT weights as 32-bit limbs (W < M < 2^111)
    unsigned int Ml[4];                  // M as 32-bit limbs
    unsigned long long Mw[2], Hw[2];     // M and floor(M / 2) as 64-bit words
    double invM;                         // 1 / M (rounded)
};

// 4 consecutive columns per thread: 4 bytes from each plane, 4 doubles out.
// S = sum_t u_t W_t is accumulated limb-wise (u_t < 2^8 times a 32-bit limb: one
// IMAD.WIDE.U32 per limb, each limb sum < 14 * 2^40); q = floor(S / M) comes from a
// double estimate (off by at most one), X = S - q M is formed limb-wise in signed
// 64-bit words and carried into a 128-bit integer, then moved into [0, M) and to
// the balanced representative in (-M/2, M/2].
template <int NM>
__global__ void __launch_bounds__(256) oz2_reconstruct_kernel(const uint8_t *__restrict__ R, int64_t ldr,
                                                              int64_t plane, const int *__restrict__ ea,
                                                              const int *__restrict__ fb, const Oz2Crt crt,
                                                              double *__restrict__ C, int64_t ldc, int64_t rows,
                                                              int64_t cols, int64_t ea_ld) {
    const __int128 M = (__int128)(((u128)crt.Mw[1] << 64) | crt.Mw[0]);
    const __int128 H = (__int128)(((u128)crt.Hw[1] << 64) | crt.Hw[0]);
    // grid-stride over (row, 4-column group); the launch covers every item once
    for (int64_t row = (int64_t)blockIdx.y * blockDim.y + threadIdx.y; row < rows;
         row += (int64_t)gridDim.y * blockDim.y)
    for (int64_t c4 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 4; c4 < cols;
         c4 += (int64_t)gridDim.x * blockDim.x * 4) {
    double acc[4] = {0, 0, 0, 0};
    for (int c = 0; c < crt.nch; ++c) {
        uint64_t a[4][4];
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int l = 0; l < 4; ++l) a[j][l] = 0;
        const uint8_t *pr = R + (int64_t)c * NM * plane + row * ldr + c4;
        uint32_t u4[NM];
#pragma unroll
        for (int t = 0; t < NM; ++t)   // all planes' loads in flight together
            u4[t] = __ldcs(reinterpret_cast<const unsigned int *>(pr + (int64_t)t * plane));   // ldr, c4 % 4 == 0
#pragma unroll
        for (int t = 0; t < NM; ++t) {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const uint32_t u = __byte_perm(u4[t], 0u, 0x4440u + j);
#pragma unroll
                for (int l = 0; l < 4; ++l) a[j][l] += (uint64_t)u * crt.W[t][l];
            }
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const double Sd = fma((double)a[j][3], 79228162514264337593543950336.0,
                                  fma((double)a[j][2], 18446744073709551616.0,
                                      fma((double)a[j][1], 4294967296.0, (double)a[j][0])));
            const uint64_t q = (uint64_t)(Sd * crt.invM);   // floor(S / M) or one off
            __int128 X = 0;
#pragma unroll
            for (int l = 3; l >= 0; --l)
                X = X * (__int128)4294967296 + (__int128)((int64_t)a[j][l] - (int64_t)(q * crt.Ml[l]));
            if (X < 0) X += M;
            if (X >= M) X -= M;
            if (X > H) X -= M;
            acc[j] += (double)(long long)(X >> 64) * 18446744073709551616.0 + (double)(uint64_t)X;
        }
    }
    const int er = ea[row * ea_ld] - 2 * crt.p;
    double *crow = C + row * ldc + c4;
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (c4 + j < cols) crow[j] = scale2(acc[j], er + fb[c4 + j]);
    }
}

// FP64-pipe CRT (the default when the plan allows it, oz2_crt_fast_ok).  The
// weights and M are split into three 39-bit pieces held as doubles, so
//   S_i = sum_t u_t w_{t,i}        (u_t < 2^8, 14 terms: every partial sum < 2^51, exact)
//   q   = rint(S / M)              (relative error ~ 2^-51 of S / M < 2^12; exact
//                                   because |X| <= B = 2^(2p + lk) <= M / (2 r) with
//                                   r >= 1 + 1/64, far from the half-integers)
//   T_i = S_i - q M_i              (|T_i| < 2^51, exact in one FMA)
//   X   = T_2 2^78 + T_1 2^39 + T_0, summed with two TwoSums: every intermediate is an
//         integer, the two error terms add exactly, so X is rounded once.
// Four FP64 operations per modulus and column (one DADD turns the byte into a double
// through the 2^52 exponent trick, three DFMAs) instead of four IMAD.WIDE plus
// 128-bit fix-ups: the integer pipes were the bottleneck of oz2_reconstruct_kernel.
struct Oz2CrtF {
    int p;
    double w[OZ2_MAX_MODULI][3];   // W_t pieces (39 bits each)
    double Mp[3];                  // M pieces
    double invM39, invM;           // 2^39 / M, 1 / M
};

// The certificate in the CRT pass for sign-uniform rows and columns (R23).
// When row i of A and column j of B each hold entries of one sign, every product
// A_ik B_kj has the same sign and D_ij = |(AB)_ij|; with the a-priori bound
// E = (sa_i + sb_j + min) / 4 + 2^-53 |X| on |X - AB 2^-(e_i+f_j-2p)| (R21) the element is
// certified when E (1 + tau) <= tau |X|, i.e. when
//   (sa_i + sb_j + min(sa_i, sb_j)) / 4 <= thr |X|,   thr = tau / (1 + tau) - 2^-52
// (rounded down; the left side is rounded up), which gives |C - AB| <= tau D_ij.  A zero
// row or column is exact.  Failing elements are flagged for K1 like the GEMM certificate;
// elements whose row or column mixes signs are the GEMM certificate's.  The column term
// sb_j (rounded up to double; -1 marks a column mixing signs) comes from the column-term
// pass.  Per row, T = (sa_i + sbmax + min) / (4 thr) rounded up (sbmax: the launch's
// largest uniform column term) certifies every element with |X| >= T by one compare; only
// the elements below it (none on benign data) read their own column term.
struct Oz2CrtCert {
    const unsigned *rsign = nullptr;   // null: no check in this pass; row sign bits (stride rsign_ld)
    long long rsign_ld = 1;
    const double *sbu = nullptr;       // column term: sb_j rounded up, -1 for a column mixing signs
    const double *rowT = nullptr;      // per row: the bound T_i (oz2_row_bound_kernel)
    const unsigned long long *sa = nullptr;
    long long sa_ld = 1;
    double thr4 = 0.0;                 // 4 thr, rounded down
    uint32_t *flags = nullptr;
    long long ldf = 0;
    uint32_t *emask = nullptr;
    long long ldw = 0;
    unsigned *fallback = nullptr;
};

__device__ __forceinline__ void two_sum(double a, double b, double &s, double &e) {
    s = a + b;
    const double bb = s - a;
    e = (a - (s - bb)) + (b - bb);
}

// 8 consecutive columns per thread: one 8-byte load per plane (all NM in flight),
// then two groups of four columns through the FP64 pieces, each stored at once.
// One K chunk (K <= 65536); longer K uses the integer pass.
template <int NM, bool CERT>
__global__ void __launch_bounds__(256, 3) oz2_crt_fp64_kernel(const uint8_t *__restrict__ R, int64_t ldr,
                                                              int64_t plane, const int *__restrict__ ea,
                                                              const int *__restrict__ fb, const Oz2CrtF crt,
                                                              double *__restrict__ C, int64_t ldc, int64_t rows,
                                                              int64_t cols, int vec, int64_t ea_ld,
                                                              const Oz2CrtCert cc) {
    const double two52 = 4503599627370496.0, two39 = 549755813888.0, two78 = 302231454903657293676544.0;
    if (CERT && blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0 && threadIdx.y == 0)
        atomicAdd(cc.fallback + 2, 1u);   // stats: CRT launches certifying sign-uniform rows / columns
    for (int64_t row = (int64_t)blockIdx.y * blockDim.y + threadIdx.y; row < rows;
         row += (int64_t)gridDim.y * blockDim.y)
    for (int64_t c16 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8; c16 < cols;
         c16 += (int64_t)gridDim.x * blockDim.x * 8) {
    const uint8_t *pr = R + row * ldr + c16;
    uint2 u16[NM];
#pragma unroll
    for (int t = 0; t < NM; ++t)   // all planes' loads in flight together (ldr, plane % 16 == 0)
        u16[t] = __ldcs(reinterpret_cast<const uint2 *>(pr + (int64_t)t * plane));
    const int er = ea[row * ea_ld] - 2 * crt.p;
    double *crow = C + row * ldc + c16;
    // R23: |X| >= T_i certifies the element by one compare (T_i: the row's bound over the
    // launch's largest uniform column term, 0 for a mixing or zero row); below it, the
    // element's own column term decides
    const double T = CERT ? cc.rowT[row] : 0.0;
    uint32_t bad = 0;
#pragma unroll
    for (int g = 0; g < 2; ++g) {
        double acc[4];
        {
            uint32_t w4[NM];
#pragma unroll
            for (int t = 0; t < NM; ++t) w4[t] = g == 0 ? u16[t].x : u16[t].y;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                double S0 = 0.0, S1 = 0.0, S2 = 0.0;
#pragma unroll
                for (int t = 0; t < NM; ++t) {
                    const double ud = __hiloint2double(0x43300000, (int)__byte_perm(w4[t], 0u, 0x4440u + j)) - two52;
                    S0 = fma(ud, crt.w[t][0], S0);
                    S1 = fma(ud, crt.w[t][1], S1);
                    S2 = fma(ud, crt.w[t][2], S2);
                }
                const double q = rint(fma(fma(S2, two39, S1), crt.invM39, S0 * crt.invM));
                const double T0 = fma(-q, crt.Mp[0], S0);
                const double T1 = fma(-q, crt.Mp[1], S1);
                const double T2 = fma(-q, crt.Mp[2], S2);
                double s1, e1, s2, e2;
                two_sum(T2 * two78, T1 * two39, s1, e1);
                two_sum(s1, T0, s2, e2);
                acc[j] = s2 + (e1 + e2);
            }
        }
        const int64_t c0 = c16 + 4 * g;
        if (CERT) {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if (fabs(acc[j]) >= T || c0 + j >= cols) continue;   // certified by the row bound
                const double sbd = cc.sbu[c0 + j];   // -1: a column mixing signs (the GEMM's); 0: exact
                if (sbd <= 0.0) continue;
                const double sad = __ull2double_ru(cc.sa[row * cc.sa_ld]);   // (T > 0: a uniform nonzero row)
                if (__dadd_ru(__dadd_ru(sad, sbd), fmin(sad, sbd)) > __dmul_rd(fabs(acc[j]), cc.thr4))
                    bad |= 1u << (4 * g + j);
            }
        }
        if (vec && c0 + 4 <= cols) {
            __stcs(reinterpret_cast<double2 *>(crow + 4 * g),
                   make_double2(scale2(acc[0], er + fb[c0]), scale2(acc[1], er + fb[c0 + 1])));
            __stcs(reinterpret_cast<double2 *>(crow + 4 * g + 2),
                   make_double2(scale2(acc[2], er + fb[c0 + 2]), scale2(acc[3], er + fb[c0 + 3])));
        } else {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (c0 + j < cols) crow[4 * g + j] = scale2(acc[j], er + fb[c0 + j]);
        }
    }
    if (CERT && bad) {   // 8 columns aligned to 8: inside one word of the element mask
        atomicOr(cc.emask + row * cc.ldw + (c16 >> 5), bad << (c16 & 31));
        uint32_t *f = cc.flags + (row >> 7) * cc.ldf + (c16 >> 7);
        if (atomicExch(f, 1u) == 0u) atomicAdd(cc.fallback, 1u);
        atomicAdd(cc.fallback + 1, (unsigned)__popc(bad));
    }
    }
}

// ------------------------------------------------------------------------
// host launchers
// ------------------------------------------------------------------------
// CTAs of the row-slicing kernels (tuning knob PDL_SPLIT_CTAS).  C4 sweep of
// oz2_split_rows: 148 / 296 / 592 / 1184 CTAs -> 4.90 / 3.11 / 2.60 / 2.41 ms with
// 2.4 / 2.4 / 3.3 / 3.5 GB DRAM read: fewer CTAs keep the second read of a row in
// L2 but lose more latency hiding than they save bandwidth.
static int split_ctas() {
    const char *e = getenv("PDL_SPLIT_CTAS");
    return e && atoi(e) > 0 ? atoi(e) : 148 * 8;
}

static cudaError_t upload_moduli(const Ozaki2Plan &P) {
    // identical for every plan (the moduli table is fixed); cheap synchronous copy
    static bool done = false;
    static int dev_done[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (done && dev < 64 && dev_done[dev]) return cudaSuccess;
    double m[OZ2_MAX_MODULI], inv[OZ2_MAX_MODULI];
    for (int t = 0; t < OZ2_MAX_MODULI; ++t) {
        m[t] = (double)kModuli[t];
        inv[t] = 1.0 / (double)kModuli[t];
    }
    int mi[OZ2_MAX_MODULI];
    for (int t = 0; t < OZ2_MAX_MODULI; ++t) mi[t] = kModuli[t];
    cudaError_t e = cudaMemcpyToSymbol(c_oz2_m, m, sizeof m);
    if (e == cudaSuccess) e = cudaMemcpyToSymbol(c_oz2_inv, inv, sizeof inv);
    if (e == cudaSuccess) e = cudaMemcpyToSymbol(c_oz2_mi, mi, sizeof mi);
    if (e == cudaSuccess && dev < 64) {
        dev_done[dev] = 1;
        done = true;
    }
    (void)P;
    return e;
}

cudaError_t launch_ozaki2_split_a(const double *A, int64_t lda, int64_t rows, int64_t K, const Ozaki2Plan &P,
                                  int8_t *A8, int *ea, cudaStream_t s, int *launches, unsigned long long *sa,
                                  int64_t lda8, int64_t ea_ld, int64_t sa_ld, unsigned *rsign) {
    if (rows <= 0) return cudaSuccess;
    if (lda8 <= 0) lda8 = P.ld8;
    cudaError_t e = upload_moduli(P);
    if (e != cudaSuccess) return e;
    if (P.check) {
        if (!sa) return cudaErrorInvalidValue;
        e = sa_ld == 1 ? cudaMemsetAsync(sa, 0, (size_t)rows * sizeof(unsigned long long), s)
                       : cudaMemset2DAsync(sa, (size_t)(sa_ld * 8), 0, sizeof(unsigned long long), (size_t)rows, s);
        if (e != cudaSuccess) return e;
    }
    const char *mode = getenv("PDL_OZ2_SPLIT");
    if (mode && !strcmp(mode, "rows") && !P.check) {
        const int blocks = (int)(rows < split_ctas() ? rows : split_ctas());
        oz2_split_rows_kernel<<<blocks, 256, 0, s>>>(A, lda, rows, K, P.n, P.p, P.Kc, P.nch, A8, lda8, ea, ea_ld);
        if (launches) *launches += 1;
        return cudaGetLastError();
    }
    oz2_rowmax_kernel<<<(unsigned)((rows + 7) / 8), 256, 0, s>>>(A, lda, rows, K, ea, ea_ld, rsign);
    const int64_t groups = (int64_t)P.nch * P.Kc / 8;
    dim3 grid((unsigned)std::min<int64_t>((groups + 255) / 256, 64), (unsigned)std::min<int64_t>(rows, 65535));
    const int vec = ((reinterpret_cast<uintptr_t>(A) & 15u) == 0 && (lda & 1) == 0) ? 1 : 0;
    oz2_residue_rows_kernel<<<grid, 256, 0, s>>>(A, lda, rows, K, P.n, P.np, P.p, P.Kc, P.nch, A8, lda8, ea, ea_ld,
                                                 vec, sa, sa_ld);
    if (launches) *launches += 2;
    return cudaGetLastError();
}

cudaError_t launch_ozaki2_split_b(const double *B, int64_t ldb, int64_t K, int64_t cols, const Ozaki2Plan &P,
                                  int8_t *Bt8, int *fb, unsigned long long *bmax, cudaStream_t s,
                                  unsigned long long *sb, unsigned *csign) {
    if (cols <= 0) return cudaSuccess;
    cudaError_t e = upload_moduli(P);
    if (e != cudaSuccess) return e;
    if (P.check) {
        if (!sb) return cudaErrorInvalidValue;
        if ((e = cudaMemsetAsync(sb, 0, (size_t)cols * sizeof(unsigned long long), s)) != cudaSuccess) return e;
    }
    e = cudaMemsetAsync(bmax, 0, (size_t)cols * sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    if (csign && (e = cudaMemsetAsync(csign, 0, (size_t)cols * sizeof(unsigned), s)) != cudaSuccess) return e;
    if (K > 0) {
        dim3 g1((unsigned)((cols + 255) / 256), (unsigned)((K + 255) / 256));
        oz2_colmax_kernel<<<g1, 256, 0, s>>>(B, ldb, K, cols, bmax, csign);
    }
    const int64_t Kpad = (int64_t)P.nch * P.Kc;
    // one k tile per CTA (C4: 1.70 ms; 4 or 16 tiles per CTA with fewer column-sum
    // atomics measured 1.87 / 1.88 ms -- many CTAs in flight keep the loads overlapped)
    const int64_t nkt = (Kpad + 63) / 64, ncb = (cols + 31) / 32;
    const int64_t gy = std::max<int64_t>(1, std::min<int64_t>(nkt, 65535));
    dim3 g2((unsigned)ncb, (unsigned)gy);
    oz2_split_cols_t_kernel<<<g2, 256, 0, s>>>(B, ldb, K, cols, P.n, P.np, P.p, P.Kc, P.nch, bmax, Bt8, P.ld8, fb,
                                               sb);
    return cudaGetLastError();
}

// The FP64-pipe CRT needs one K chunk, M < 2^117 (three 39-bit pieces) and a clear gap between
// the largest valid |X| (B = 2^(2p + ceil(log2 Kc))) and M / 2: M >= 2 B (1 + 1/64).
// Holds for every plan of 2..14 moduli (M / 2^floor(log2 M) >= 1.029).
bool oz2_crt_fast_ok(const Ozaki2Plan &P) {
    const u128 M = ((u128)P.Mw[1] << 64) | P.Mw[0];
    if (P.n < 2 || P.nch != 1 || (M >> 117) != 0) return false;
    const int e = 2 * P.p + ilog2_ceil(P.Kc < 1 ? 1 : P.Kc);
    if (e + 1 >= 127) return false;
    const u128 twoB = (u128)1 << (e + 1);
    return M >= twoB + (twoB >> 6);
}

cudaError_t launch_ozaki2_reconstruct(const uint8_t *R, int64_t ldr, int64_t plane, const int *ea, const int *fb,
                                      const Ozaki2Plan &P, double *C, int64_t ldc, int64_t rows, int64_t cols,
                                      cudaStream_t s, int64_t ea_ld, const Oz2Guard *guard) {
    if (rows <= 0 || cols <= 0) return cudaSuccess;
    if ((reinterpret_cast<uintptr_t>(R) & 3u) || (ldr & 3) || (plane & 3)) return cudaErrorInvalidValue;
    const char *crt_mode = getenv("PDL_OZ2_CRT");
    if (oz2_crt_fast_ok(P) && !(crt_mode && !strcmp(crt_mode, "int"))) {
        Oz2CrtF f;
        f.p = P.p;
        const u128 mask = ((u128)1 << 39) - 1;
        for (int t = 0; t < OZ2_MAX_MODULI; ++t) {
            const u128 W = ((u128)P.W[t][1] << 64) | P.W[t][0];
            for (int i = 0; i < 3; ++i) f.w[t][i] = (double)(unsigned long long)((W >> (39 * i)) & mask);
        }
        const u128 M = ((u128)P.Mw[1] << 64) | P.Mw[0];
        for (int i = 0; i < 3; ++i) f.Mp[i] = (double)(unsigned long long)((M >> (39 * i)) & mask);
        f.invM39 = 549755813888.0 / P.Md;
        f.invM = 1.0 / P.Md;
        if ((reinterpret_cast<uintptr_t>(R) & 15u) || (ldr & 15) || (plane & 15)) return cudaErrorInvalidValue;
        const int vec = ((reinterpret_cast<uintptr_t>(C) & 15u) == 0 && (ldc & 1) == 0) ? 1 : 0;
        Oz2CrtCert cc;
        if (guard && guard->rsign) {   // R23: the certificate of sign-uniform rows / columns
            if (!guard->sbu || !guard->rowT || !guard->sa || !guard->flags || !guard->emask || !guard->fallback)
                return cudaErrorInvalidValue;
            cc.rowT = guard->rowT;
            cc.rsign = guard->rsign;
            cc.rsign_ld = guard->rsign_ld;
            cc.sbu = guard->sbu;
            cc.sa = guard->sa;
            cc.sa_ld = guard->sa_ld;
            cc.thr4 = oz2_uniform_thr4(guard->tau);
            cc.flags = guard->flags;
            cc.ldf = guard->ldf;
            cc.emask = guard->emask;
            cc.ldw = guard->ldw;
            cc.fallback = guard->fallback;
        }
        dim3 block(32, 8);
        dim3 grid((unsigned)((cols + 255) / 256), (unsigned)std::min<int64_t>((rows + 7) / 8, 65535));
        switch (P.n) {
#define OZ2_CASE(k) \
    case k:                                                                                              \
        if (cc.rsign)                                                                                    \
            oz2_crt_fp64_kernel<k, true><<<grid, block, 0, s>>>(R, ldr, plane, ea, fb, f, C, ldc, rows, cols, \
                                                                vec, ea_ld, cc);                         \
        else                                                                                             \
            oz2_crt_fp64_kernel<k, false><<<grid, block, 0, s>>>(R, ldr, plane, ea, fb, f, C, ldc, rows,      \
                                                                 cols, vec, ea_ld, cc);                  \
        break;
            OZ2_CASE(2) OZ2_CASE(3) OZ2_CASE(4) OZ2_CASE(5) OZ2_CASE(6) OZ2_CASE(7) OZ2_CASE(8) OZ2_CASE(9)
            OZ2_CASE(10) OZ2_CASE(11) OZ2_CASE(12) OZ2_CASE(13) OZ2_CASE(14)
#undef OZ2_CASE
            default: return cudaErrorInvalidValue;
        }
        return cudaGetLastError();
    }
    Oz2Crt crt;
    crt.n = P.n;
    crt.nch = P.nch;
    crt.p = P.p;
    for (int t = 0; t < OZ2_MAX_MODULI; ++t)
        for (int l = 0; l < 4; ++l) crt.W[t][l] = (unsigned int)(P.W[t][l >> 1] >> (32 * (l & 1)));
    for (int l = 0; l < 4; ++l) crt.Ml[l] = (unsigned int)(P.Mw[l >> 1] >> (32 * (l & 1)));
    crt.Mw[0] = P.Mw[0];
    crt.Mw[1] = P.Mw[1];
    crt.Hw[0] = P.Hw[0];
    crt.Hw[1] = P.Hw[1];
    crt.invM = 1.0 / P.Md;
    dim3 block(32, 8);
    dim3 grid((unsigned)((cols + 127) / 128), (unsigned)((rows + 7) / 8));
    switch (P.n) {
#define OZ2_CASE(k) \
    case k: oz2_reconstruct_kernel<k><<<grid, block, 0, s>>>(R, ldr, plane, ea, fb, crt, C, ldc, rows, cols, ea_ld); break;
        OZ2_CASE(2) OZ2_CASE(3) OZ2_CASE(4) OZ2_CASE(5) OZ2_CASE(6) OZ2_CASE(7) OZ2_CASE(8) OZ2_CASE(9) OZ2_CASE(10)
        OZ2_CASE(11) OZ2_CASE(12) OZ2_CASE(13) OZ2_CASE(14)
#undef OZ2_CASE
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

}  // namespace pdlk
