"""CPU pin of the split arithmetic of the FP32 task variant "tf32bf16" (R22).

    a = a_hi + a_lo exactly,  a_hi = rn_tf32(a) (11 significant bits), a_lo = a - a_hi
    a*b ~= a_hi*b_hi + rn_bf16(a_hi)*rn_bf16(b_lo) + rn_bf16(a_lo)*rn_bf16(b_hi)

The dropped a_lo*b_lo is <= 2^-22 |a||b|; each correction product carries two BF16
roundings (<= 2^-8 relative each) of a product <= 2^-11 |a||b|, so the split error is
at most (2^-17 + 2^-22)(1 + 2^-10) |a||b| per product and, summed over k, per element
of C relative to D = |A||B| (R13).  These tests emulate the roundings with exact
integer bit operations on float32 patterns (independent of the CUDA path) and check
that bound on random, structured worst-case and adversarial inputs, and that small
integers split exactly (the bitwise GPU pins rely on it).
"""
import numpy as np

import oracle

BOUND = (2.0 ** -17 + 2.0 ** -22) * (1 + 2.0 ** -10)


def rna_tf32(x):
    """Round to nearest, ties away from zero, keeping 10 explicit mantissa bits
    (cvt.rna.tf32.f32 on finite inputs)."""
    b = np.asarray(x, np.float32).view(np.uint32).astype(np.uint64)
    b = (b + 0x1000) & 0xFFFFE000
    return b.astype(np.uint32).view(np.float32)


def rn_bf16(x):
    """Round to nearest even to 7 explicit mantissa bits (cvt.rn.bf16.f32)."""
    b = np.asarray(x, np.float32).view(np.uint32).astype(np.uint64)
    lsb = (b >> 16) & 1
    b = (b + 0x7FFF + lsb) & 0xFFFF0000
    return b.astype(np.uint32).view(np.float32)


def split(x):
    x = np.asarray(x, np.float32)
    hi = rna_tf32(x)
    lo = (x - hi).astype(np.float32)   # exact: hi is x rounded to 11 bits
    return hi, rn_bf16(hi), rn_bf16(lo)


def mixed_product(a, b):
    ah, ahb, alb = split(a)
    bh, bhb, blb = split(b)
    f = np.float64
    return ah.astype(f) * bh.astype(f) + ahb.astype(f) * blb.astype(f) + alb.astype(f) * bhb.astype(f)


def mixed_matmul(A, B):
    ah, ahb, alb = (p.astype(np.float64) for p in split(A))
    bh, bhb, blb = (p.astype(np.float64) for p in split(B))
    return ah @ bh + ahb @ blb + alb @ bhb


def test_roundings_match_their_definitions():
    # tf32: 1 + 2^-11 is a tie -> away from zero; 1 + 2^-11 + 2^-12 -> up
    assert rna_tf32(np.float32(1 + 2.0 ** -11)) == np.float32(1 + 2.0 ** -10)
    assert rna_tf32(np.float32(-(1 + 2.0 ** -11))) == np.float32(-(1 + 2.0 ** -10))
    assert rna_tf32(np.float32(1 + 2.0 ** -12)) == np.float32(1.0)
    # bf16: ties to even
    assert rn_bf16(np.float32(1 + 2.0 ** -8)) == np.float32(1.0)
    assert rn_bf16(np.float32(1 + 3 * 2.0 ** -8)) == np.float32(1 + 2.0 ** -6)
    assert rn_bf16(np.float32(1 + 2.0 ** -8 + 2.0 ** -20)) == np.float32(1 + 2.0 ** -7)


def test_split_is_exact_for_the_hi_lo_identity():
    rng = np.random.default_rng(1)
    x = (rng.standard_normal(100000) * 2.0 ** rng.integers(-40, 40, 100000)).astype(np.float32)
    hi = rna_tf32(x)
    lo = (x - hi).astype(np.float32)
    assert np.array_equal(hi.astype(np.float64) + lo.astype(np.float64), x.astype(np.float64))
    assert np.all(np.abs(lo.astype(np.float64)) <= 2.0 ** -11 * np.abs(x.astype(np.float64)))


def test_small_integers_split_exactly():
    x = np.arange(-256, 257, dtype=np.float32)
    hi, hb, lb = split(x)
    assert np.array_equal(hi, x) and np.array_equal(hb, x) and not lb.any()
    a, b = np.meshgrid(np.arange(-16, 17), np.arange(-16, 17))
    assert np.array_equal(mixed_product(a.astype(np.float32), b.astype(np.float32)), (a * b).astype(np.float64))


def _rel_err(a, b):
    p = a.astype(np.float64) * b.astype(np.float64)
    return np.abs(mixed_product(a, b) - p) / np.abs(p)


def test_per_product_bound_random():
    rng = np.random.default_rng(2)
    a = (rng.random(1 << 20) + 0.5).astype(np.float32) * np.float32(2.0) ** rng.integers(-20, 20, 1 << 20)
    b = (rng.random(1 << 20) - 0.5).astype(np.float32) * np.float32(2.0) ** rng.integers(-20, 20, 1 << 20)
    e = _rel_err(a.astype(np.float32), b.astype(np.float32))
    assert e.max() <= BOUND
    assert e.max() > 2.0 ** -19   # the bound is approached (the correction roundings are real)


def test_per_product_bound_structured_worst_case():
    """Every mantissa pattern class that drives the four BF16 roundings to (near)
    their maximum: hi bits 8-10 = 100 (a tie at bit 8 of hi) or 011/101, lo as
    large as RN-to-11-bits allows with its own rounding bit pattern at a BF16 tie."""
    vals = []
    for hi_tail in (0b011, 0b100, 0b101, 0b111):
        for lo_pat in range(0, 1 << 13, 37):
            m = (np.uint32(0x3F800000) | np.uint32((hi_tail << 13) | lo_pat) | np.uint32(0x7F << 16))
            vals.append(m)
    x = np.array(vals, np.uint32).view(np.float32)
    a = np.repeat(x, x.size)
    b = np.tile(x, x.size)
    e = _rel_err(a, b)
    assert e.max() <= BOUND


def test_elementwise_bound_against_the_oracle():
    """Summed over k with fp64 accumulation (the split error alone), against the
    CPU oracle: |C - AB| <= BOUND * D element by element, on signed data with
    cancellation and on rows/columns spread over 2^+-30."""
    rng = np.random.default_rng(3)
    A = (rng.random((64, 300)) * 2 - 1).astype(np.float32)
    B = (rng.random((300, 48)) * 2 - 1).astype(np.float32)
    A[:, 1] = -A[:, 0]
    B[1] = B[0]
    A *= (2.0 ** rng.integers(-30, 30, (64, 1))).astype(np.float32)
    B *= (2.0 ** rng.integers(-30, 30, (1, 48))).astype(np.float32)
    C = mixed_matmul(A, B)
    Cref, D = oracle.matmul(A, B)
    err = oracle.scaled_error(C, Cref, D)
    assert err.max() <= BOUND + 2.0 ** -50
