"""Pins for the CPU oracle, CPU only.

Each pin ties oracle/ to something other than itself: exact integer
arithmetic through numpy's int64 matmul (a library routine on a special case
where the product is exact), exact rational arithmetic (fractions.Fraction),
closed forms (identity, permutation, rank-1, K=1, K=0) and the classical
gamma_K forward-error bound of recursive summation (Higham, Accuracy and
Stability of Numerical Algorithms, Thm 3.5 / eq. 3.13).  A dropped term, a sign
error, a wrong index or a transposed operand in oracle.c fails at least one of
these.  The paper prints no DGEMM output, so parity with the paper itself is
unpinned (Figure 5 values missing).
"""
from fractions import Fraction

import numpy as np
import pytest

import oracle
import workloads as W

TINY = [1, 2, 3, 5, 7, 8, 13, 17, 31, 32, 33]
EDGE = [127, 128, 129]


def _int_exact(A_int, B_int):
    # exact integer product (entries small enough that int64 never overflows)
    return A_int.astype(np.int64) @ B_int.astype(np.int64)


@pytest.mark.parametrize("M,N,K", [(m, n, k) for m in (1, 3, 8, 17) for n in (1, 5, 13, 32)
                                   for k in (1, 2, 7, 33)] + [(e, e, e) for e in EDGE])
def test_p1_dyadic_exact_vs_integer_matmul(M, N, K):
    """P1: dyadic inputs k/2^8 -> every partial sum is exact in double, so the
    oracle must equal the exact integer product scaled by 2^-16, bitwise."""
    A = W.dyadic((M, K), np.float64, 11 + M)
    B = W.dyadic((K, N), np.float64, 13 + N)
    exact = _int_exact(A * 256, B * 256).astype(np.float64) / 65536.0
    C, D = oracle.matmul(A, B)
    assert np.array_equal(C, exact)
    Dexact = _int_exact(np.abs(A) * 256, np.abs(B) * 256).astype(np.float64) / 65536.0
    assert np.array_equal(D, Dexact)


def test_p1_fraction_bruteforce_tiny():
    """P1 with exact rationals on U[0,1) doubles: |Cref - exact| <= gamma_K * D."""
    for (M, N, K) in [(3, 4, 5), (7, 2, 31), (2, 3, 129)]:
        A = W.uniform((M, K), np.float64, 5 + K)
        B = W.signed((K, N), np.float64, 6 + K)
        C, D = oracle.matmul(A, B)
        u = Fraction(1, 2 ** 53)
        gamma = K * u / (1 - K * u)
        for i in range(M):
            for j in range(N):
                ex = sum((Fraction(float(A[i, k])) * Fraction(float(B[k, j])) for k in range(K)),
                         Fraction(0))
                dex = sum((abs(Fraction(float(A[i, k])) * Fraction(float(B[k, j])))
                           for k in range(K)), Fraction(0))
                assert abs(Fraction(float(C[i, j])) - ex) <= gamma * dex
                assert abs(Fraction(float(D[i, j])) - dex) <= gamma * dex


@pytest.mark.parametrize("M,K", [(5, 5), (17, 33), (33, 8), (129, 127)])
def test_p2_identity(M, K):
    """P2: A.I = A and I.B = B bitwise (products with 0/1 and sums with 0 are exact)."""
    A = W.signed((M, K), np.float64, 21)
    C, _ = oracle.matmul(A, W.identity(K, K, np.float64))
    assert np.array_equal(C, A)
    C2, _ = oracle.matmul(W.identity(M, M, np.float64), A)
    assert np.array_equal(C2, A)
    # rectangular identity picks the leading columns
    Ir = W.identity(K, 3, np.float64)
    C3, _ = oracle.matmul(A, Ir)
    assert np.array_equal(C3, A[:, :3])


@pytest.mark.parametrize("n,m", [(7, 3), (32, 17), (65, 9)])
def test_p3_permutation(n, m):
    """P3: P.B permutes rows of B; A.P permutes columns of A (bitwise)."""
    P, p = W.permutation(n, np.float64, 31 + n)
    B = W.signed((n, m), np.float64, 32)
    C, _ = oracle.matmul(P, B)
    assert np.array_equal(C, B[p, :])
    A = W.signed((m, n), np.float64, 33)
    C2, _ = oracle.matmul(A, P)
    inv = np.empty_like(p)
    inv[p] = np.arange(n)
    assert np.array_equal(C2, A[:, inv])


@pytest.mark.parametrize("M,N,K", [(9, 11, 13), (33, 17, 64), (128, 129, 257)])
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_p4_rank1_closed_form(M, N, K, dt):
    """P4: A = u v^T, B = x y^T (integers in [-4,4]) -> C = (v.x) u y^T exactly."""
    u, v = W.rank1_factors(M, K, 41)
    x, y = W.rank1_factors(K, N, 42)
    A = np.outer(u, v).astype(dt)
    B = np.outer(x, y).astype(dt)
    s = int(np.dot(v, x))
    expect = (s * np.outer(u, y)).astype(np.float64)
    C, _ = oracle.matmul(A, B)
    assert np.array_equal(C, expect)


def test_p5_integer_matrices():
    """P5: integer entries in {-8..8}: exact, equals int64 matmul bitwise."""
    for (M, N, K) in [(31, 33, 64), (64, 17, 129)]:
        for dt in (np.float64, np.float32):
            A = W.integers((M, K), dt, 51)
            B = W.integers((K, N), dt, 52)
            C, _ = oracle.matmul(A, B)
            assert np.array_equal(C, _int_exact(A, B).astype(np.float64))


def test_p6_k1_outer_product():
    """P6: K = 1 -> C_ij = fl(a_i * b_j), one rounding (numpy's multiply.outer)."""
    a = W.signed((19, 1), np.float64, 61)
    b = W.signed((1, 23), np.float64, 62)
    C, D = oracle.matmul(a, b)
    assert np.array_equal(C, np.multiply.outer(a[:, 0], b[0, :]))
    assert np.array_equal(D, np.abs(C))


def test_k0_empty_sum_and_empty_shapes():
    A = np.zeros((4, 0))
    B = np.zeros((0, 5))
    C, D = oracle.matmul(A, B)
    assert C.shape == (4, 5) and np.all(C == 0) and np.all(D == 0)
    C, _ = oracle.matmul(np.zeros((0, 3)), np.zeros((3, 2)))
    assert C.shape == (0, 2)


def test_p8_error_bound_random():
    """P8: U[0,1) doubles at K=600: sampled elements within gamma_K * D of the
    exact rational value (Fraction), D == Cref for non-negative inputs."""
    M, N, K = 6, 5, 600
    A = W.uniform((M, K), np.float64, 71)
    B = W.uniform((K, N), np.float64, 72)
    C, D = oracle.matmul(A, B)
    assert np.array_equal(C, D)            # non-negative: |A||B| is the same sum
    u = Fraction(1, 2 ** 53)
    gamma = K * u / (1 - K * u)
    for (i, j) in [(0, 0), (5, 4), (3, 2)]:
        ex = sum((Fraction(float(A[i, k])) * Fraction(float(B[k, j])) for k in range(K)),
                 Fraction(0))
        assert abs(Fraction(float(C[i, j])) - ex) <= gamma * ex


def test_float32_inputs_promoted_exactly():
    """float32 inputs are promoted exactly: same result as the float64 copy."""
    A = W.uniform((17, 40), np.float32, 81)
    B = W.uniform((40, 9), np.float32, 82)
    C32, D32 = oracle.matmul(A, B)
    C64, D64 = oracle.matmul(A.astype(np.float64), B.astype(np.float64))
    assert np.array_equal(C32, C64) and np.array_equal(D32, D64)


def test_rows_subset_and_threads_invariance():
    A = W.signed((50, 70), np.float64, 91)
    B = W.signed((70, 30), np.float64, 92)
    C, D = oracle.matmul(A, B, nthreads=1)
    Cm, Dm = oracle.matmul(A, B, nthreads=4)
    assert np.array_equal(C, Cm) and np.array_equal(D, Dm)
    rows = [49, 0, 7, 7, 31]
    Cs, Ds = oracle.matmul(A, B, rows=rows)
    assert np.array_equal(Cs, C[rows]) and np.array_equal(Ds, D[rows])
    # D is the oracle of |A| |B| and bounds |C|
    Dabs, _ = oracle.matmul(np.abs(A), np.abs(B))
    assert np.array_equal(D, Dabs)
    assert np.all(np.abs(C) <= D)


def test_nonfinite_propagates():
    A = W.uniform((4, 6), np.float64, 1)
    B = W.uniform((6, 3), np.float64, 2)
    A[2, 3] = np.nan
    C, _ = oracle.matmul(A, B)
    assert np.all(np.isnan(C[2])) and np.all(np.isfinite(np.delete(C, 2, axis=0)))


def test_scaled_error_metric():
    Cref = np.array([[1.0, 0.0, -2.0]])
    D = np.array([[1.0, 0.0, 4.0]])
    err = oracle.scaled_error(np.array([[1.0 + 1e-6, 0.0, -2.0]]), Cref, D)
    assert err[0, 0] == pytest.approx(1e-6) and err[0, 1] == 0 and err[0, 2] == 0
    err = oracle.scaled_error(np.array([[1.0, 1e-300, np.nan]]), Cref, D)
    assert np.isinf(err[0, 1]) and np.isinf(err[0, 2])


def test_bad_arguments_rejected():
    with pytest.raises(ValueError):
        oracle.matmul(np.zeros((2, 3)), np.zeros((4, 2)))
    with pytest.raises(RuntimeError):
        oracle.matmul(np.zeros((2, 3)), np.zeros((3, 2)), rows=[2])
