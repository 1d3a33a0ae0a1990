"""GPU parity of the FP32 task variants (SGEMM_VARIANT): "tf32bf16" (the default,
DESIGN.md R22) -- a_hi*b_hi on kind::tf32 plus the two correction products
a_hi'*b_lo' + a_lo'*b_hi' on kind::f16 with BF16 operands, two TF32-equivalent tensor
passes per K block -- and "3xtf32" (three kind::tf32 products, selectable).  The
shape / pin tests run for both (fixture `props`); test_gpu_parity.py covers the
default through the plain descriptor.

The bar is the north star's FP32 one: max element-wise error 1e-5 scaled by
D = |A||B| (R13) against the CPU oracle (fp64 triple loop).  R22 bounds the
tf32bf16 split error by (2^-17 + 2^-22)(1 + 2^-10) D ~ 7.9e-6 D per element on any
finite input (largest per-product error found: 4.6e-6; the bound is pinned on the
CPU in tests/test_tf32bf16_bound.py); the accumulation in TMEM adds the K-chunked
promotion error of R16.  Exact-arithmetic pins (small integers:
hi = x, lo = 0, exactly representable in BF16 and TF32) are bitwise.
"""
import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402

TOL = 1e-5
VARIANT = {"SGEMM_VARIANT": "tf32bf16"}


@pytest.fixture(params=["tf32bf16", "3xtf32"])
def props(request):
    return {"SGEMM_VARIANT": request.param}


@pytest.fixture(autouse=True)
def _env(monkeypatch):
    monkeypatch.delenv("PDL_DRY_RUN", raising=False)
    monkeypatch.delenv("PDL_SGEMM_VARIANT", raising=False)
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    pdl.unload()
    yield
    pdl.unload()


def mm(A, B, tile=0, workers=1, host=False, props=VARIANT):
    pdl.load(pdl.descriptor_xml(workers, props=props))
    try:
        M, N = A.shape[0], B.shape[1]
        if host:
            C = np.full((M, N), np.nan, dtype=np.float32)
            pdl.task_matmul(A, B, C, tile=tile)
            pdl.run()
            return C
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        dC = torch.full((M, N), float("nan"), dtype=torch.float32, device="cuda")
        pdl.task_matmul(dA, dB, dC, tile=tile)
        pdl.run()
        return dC.cpu().numpy()
    finally:
        pdl.unload()


def check(C, A, B, rows=None, tol=TOL):
    Cref, D = oracle.matmul(A, B, rows=rows)
    Cs = C if rows is None else C[rows]
    err = oracle.scaled_error(Cs, Cref, D)
    assert np.isfinite(err).all(), "non-finite or wrong-zero outputs"
    assert err.max() <= tol, f"max scaled err {err.max():.3e} > {tol:g}"
    return err


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_configs_full_parity(name, props):
    c = W.CONFIGS[name]
    A, B = W.config_inputs(name, np.float32)
    check(mm(A, B, tile=c.tile, props=props), A, B)


@pytest.mark.parametrize("M,N,K", [(1, 1, 1), (3, 5, 7), (8, 13, 17), (33, 31, 32), (127, 129, 128),
                                   (129, 255, 257), (257, 130, 33), (200, 17, 1000), (300, 520, 95)])
def test_brute_force_shapes_host_and_device(M, N, K, props):
    A = W.signed((M, K), np.float32, 100 + M)
    B = W.signed((K, N), np.float32, 200 + N)
    check(mm(A, B, tile=32, props=props), A, B)
    check(mm(A, B, host=True, props=props), A, B)


def test_rank1_closed_form_bitwise(props):
    M, N, K = 300, 260, 520
    u, v = W.rank1_factors(M, K, 5)
    x, y = W.rank1_factors(K, N, 6)
    A = np.outer(u, v).astype(np.float32)
    B = np.outer(x, y).astype(np.float32)
    expect = (int(np.dot(v, x)) * np.outer(u, y)).astype(np.float32)
    assert np.array_equal(mm(A, B, tile=64, props=props), expect)


def test_integer_matrices_bitwise(props):
    A = W.integers((190, 300), np.float32, 7)
    B = W.integers((300, 170), np.float32, 8)
    Cref, _ = oracle.matmul(A, B)
    assert np.array_equal(mm(A, B, props=props).astype(np.float64), Cref)


def test_worker_count_and_tile_invariance_bitwise(props):
    A = W.uniform((515, 390), np.float32, 11)
    B = W.uniform((390, 333), np.float32, 12)
    ref = mm(A, B, props=props)
    check(ref, A, B)
    for workers, tile in ((2, 64), (4, 32), (8, 128), (8, 0)):
        assert np.array_equal(mm(A, B, tile=tile, workers=workers, props=props), ref), (workers, tile)


@pytest.mark.parametrize("M,N,K", [(1000, 1000, 300), (1100, 700, 513), (300, 2000, 1029)])
def test_cta_shapes_bitwise(monkeypatch, M, N, K, props):
    """1-SM and CTA-pair kernels of the variant, and the pair kernel's two K-block
    widths (PDL_K2_BK 16: SWIZZLE_64B, 7 stages; 32: SWIZZLE_128B, 3 stages): same K
    chunks, same MMA order per 16-wide K step, so bitwise the same C."""
    A = W.signed((M, K), np.float32, 63)
    B = W.signed((K, N), np.float32, 64)
    out = {}
    for v, bk in (("2sm", "16"), ("2sm", "32"), ("1sm", "16")):
        monkeypatch.setenv("PDL_K2", v)
        monkeypatch.setenv("PDL_K2_BK", bk)
        out[v + bk] = mm(A, B, props=props)
    monkeypatch.delenv("PDL_K2")
    monkeypatch.delenv("PDL_K2_BK")
    check(out["1sm16"], A, B)
    assert np.array_equal(out["1sm16"], out["2sm16"])
    assert np.array_equal(out["2sm32"], out["2sm16"])   # 7-stage SW64 ring vs 3-stage SW128 ring


def test_default_fp32_variant_is_tf32bf16():
    """A descriptor without SGEMM_VARIANT runs tf32bf16 (bitwise the explicit one)."""
    A = W.signed((300, 777), np.float32, 33)
    B = W.signed((777, 260), np.float32, 34)
    assert np.array_equal(mm(A, B, props=None), mm(A, B))


def test_differs_from_3xtf32_and_both_hold_the_bar():
    """The variant really runs (it is not the 3xTF32 kernel under another name):
    on U[-1,1) data the two give different bits, both within the bar."""
    A = W.signed((400, 2048), np.float32, 31)
    B = W.signed((2048, 300), np.float32, 32)
    c_mix = mm(A, B)
    c_3x = mm(A, B, props={"SGEMM_VARIANT": "3xtf32"})
    check(c_mix, A, B)
    check(c_3x, A, B)
    assert not np.array_equal(c_mix, c_3x)


def test_k_sweep_accuracy(capsys):
    rows = []
    for K in (256, 1024, 4096, 16384):
        A = W.uniform((256, K), np.float32, 21)
        B = W.uniform((K, 256), np.float32, 22)
        C = mm(A, B)
        Cref, D = oracle.matmul(A, B)
        err = oracle.scaled_error(C, Cref, D)
        rows.append((K, float(err.max())))
    with capsys.disabled():
        for K, mx in rows:
            print(f"\n[tf32bf16 K-sweep] K={K:6d} max_err={mx:.3e}")
    assert max(r[1] for r in rows) <= TOL


def test_adversarial_split_rounding(props):
    """Inputs whose BF16 roundings of hi and lo are all near their worst case
    (mantissas just below a BF16 rounding boundary, same sign, so nothing
    cancels) and signed K = 2..16 rows with exact cancellation partners: the
    per-element split bound of R22 (<= 7.9e-6 D) keeps them under the 1e-5 bar."""
    rng = np.random.default_rng(77)
    # x = 1 + m 2^-7 + (2^-8 - 2^-20): hi keeps 10 explicit bits, hi' rounds by ~2^-8 relative
    m = rng.integers(0, 128, size=(256, 512))
    A = (1.0 + m * 2.0 ** -7 + 2.0 ** -8 - 2.0 ** -20).astype(np.float32)
    B = (1.0 + rng.integers(0, 128, size=(512, 200)) * 2.0 ** -7 + 2.0 ** -8 - 2.0 ** -20).astype(np.float32)
    check(mm(A, B, props=props), A, B)
    for K in (2, 3, 8, 16):
        a = W.signed((64, K), np.float32, 500 + K)
        b = W.signed((K, 48), np.float32, 600 + K)
        a[:, 1] = -a[:, 0] * np.float32(1.0 + 2.0 ** -12)   # near-cancelling pair
        b[1] = b[0]
        check(mm(a, b, props=props), a, b)


def test_spread_exponents(props):
    """Rows and columns scaled over 2^+-30 (the split is per element, so the
    D-scaled error is unchanged)."""
    rng = np.random.default_rng(5)
    A = (W.signed((300, 700), np.float32, 41) * (2.0 ** rng.integers(-30, 30, size=(300, 1)))).astype(np.float32)
    B = (W.signed((700, 260), np.float32, 42) * (2.0 ** rng.integers(-30, 30, size=(1, 260)))).astype(np.float32)
    check(mm(A, B, props=props), A, B)


def test_local_chunk_tasks_reuse_b_bitwise():
    """Row-chunk tasks with PDL_TASK_REUSE_B reproduce the single task bitwise,
    and a B prepared by the 3xTF32 split is never reused by this variant."""
    M, N, K = 700, 520, 390
    A = W.uniform((M, K), np.float32, 401)
    B = W.uniform((K, N), np.float32, 402)
    pdl.load(pdl.descriptor_xml(1, props=VARIANT))
    try:
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        ref = torch.empty((M, N), dtype=torch.float32, device="cuda")
        pdl.task_matmul(dA, dB, ref)
        pdl.run()
        out = torch.full((M, N), float("nan"), dtype=torch.float32, device="cuda")
        for i, (lo, hi) in enumerate([(0, 256), (256, 300), (300, 700)]):
            pdl.task_matmul(dA[lo:hi], dB, out[lo:hi], local=True, reuse_b=i > 0)
            pdl.run()
        assert torch.equal(out, ref)
    finally:
        pdl.unload()
    check(ref.cpu().numpy(), A, B)


def test_prepared_a_rows_bitwise():
    """PDL_TASK_PREP_A of this variant (TF32 hi + BF16 [hi' | lo'] rows, the unit
    the multi-rank exchange moves) then PDL_TASK_PREPARED_A tasks: bitwise the
    plain task."""
    M, N, K = 600, 333, 700
    A = W.signed((M, K), np.float32, 71)
    B = W.signed((K, N), np.float32, 72)
    pdl.load(pdl.descriptor_xml(1, props=VARIANT))
    try:
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        ref = torch.empty((M, N), dtype=torch.float32, device="cuda")
        pdl.task_matmul(dA, dB, ref)
        pdl.run()
        pb, raw = pdl.prepared_a_info(torch.float32, K)
        assert pb > 0 and not raw
        prep = torch.empty((M, pb), dtype=torch.uint8, device="cuda")
        pdl.prepare_a(dA, prep)
        pdl.run()
        out = torch.full((M, N), float("nan"), dtype=torch.float32, device="cuda")
        for i, (lo, hi) in enumerate([(0, 300), (300, 600)]):
            pdl.task_matmul_prepared(prep[lo:hi], dB, out[lo:hi], M=hi - lo, N=N, K=K, ldb=N, ldc=N,
                                     reuse_b=i > 0)
            pdl.run()
        assert torch.equal(out, ref)
    finally:
        pdl.unload()


def test_dynamic_distribution_bitwise():
    A = W.uniform((900, 400), np.float32, 81)
    B = W.uniform((400, 700), np.float32, 82)
    ref = mm(A, B, tile=128, workers=2)
    pdl.load(pdl.descriptor_xml(2, props=VARIANT))
    try:
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        dC = torch.full((900, 700), float("nan"), dtype=torch.float32, device="cuda")
        pdl.task_matmul(dA, dB, dC, tile=128, dist="DYNAMIC")
        pdl.run()
        assert np.array_equal(dC.cpu().numpy(), ref)
    finally:
        pdl.unload()


def test_unknown_sgemm_variant_is_rejected():
    A = W.uniform((64, 64), np.float32, 1)
    pdl.load(pdl.descriptor_xml(1, props={"SGEMM_VARIANT": "tf16"}))
    try:
        dA = torch.from_numpy(A).cuda()
        dC = torch.empty((64, 64), dtype=torch.float32, device="cuda")
        pdl.task_matmul(dA, dA, dC)
        with pytest.raises(pdl.PDLError) as ei:
            pdl.run()
        assert ei.value.code == pdl.PDL_EINVAL
    finally:
        pdl.unload()


@pytest.mark.slow
def test_c4_full_size_sampled():
    """C4 16384^3 at full size in the bench's launch configuration; sampled rows
    against the oracle (every 128-row CTA band boundary class is covered by the
    random rows across the 64 pair-tile rows)."""
    c = W.CONFIGS["C4"]
    A, B = W.config_inputs("C4", np.float32)
    C = mm(A, B, tile=c.tile)
    rows = W.sampled_rows(c.M, (), c.tile, n_random=64)
    check(C, A, B, rows=rows)


def test_prepared_b_is_not_shared_between_variants(monkeypatch):
    """The prepared-B cache (PDL_TASK_REUSE_B) keys on the task variant: a B split for
    tf32bf16 (TF32 hi + BF16 pairs) is not read by a 3xtf32 task asking for reuse (TF32
    hi/lo in the same buffers), and vice versa -- C equals a fresh run of each variant."""
    M, N, K = 500, 390, 700
    A = W.signed((M, K), np.float32, 91)
    B = W.signed((K, N), np.float32, 92)
    fresh = {v: mm(A, B, props={"SGEMM_VARIANT": v}) for v in ("tf32bf16", "3xtf32")}
    assert not np.array_equal(fresh["tf32bf16"], fresh["3xtf32"])
    pdl.load(pdl.descriptor_xml(1))
    try:
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        out = torch.empty((M, N), dtype=torch.float32, device="cuda")
        for first, second in (("tf32bf16", "3xtf32"), ("3xtf32", "tf32bf16")):
            monkeypatch.setenv("PDL_SGEMM_VARIANT", first)
            pdl.task_matmul(dA, dB, out, local=True)
            pdl.run()
            assert np.array_equal(out.cpu().numpy(), fresh[first])
            monkeypatch.setenv("PDL_SGEMM_VARIANT", second)
            pdl.task_matmul(dA, dB, out, local=True, reuse_b=True)
            pdl.run()
            assert np.array_equal(out.cpu().numpy(), fresh[second])
    finally:
        pdl.unload()


@pytest.mark.parametrize("dist", ["uniform", "signed"])
def test_long_k_2_pow_20(props, dist):
    """Long-K edge for FP32: K = 2^20 + 3 (8192 promoted 128-wide chunks summed in FP32
    registers with round-to-nearest, a ragged last K block) on a small ragged C; the
    1e-5 bar holds for both variants."""
    M, N, K = 70, 37, (1 << 20) + 3
    gen = W.uniform if dist == "uniform" else W.signed
    A = gen((M, K), np.float32, 83)
    B = gen((K, N), np.float32, 84)
    check(mm(A, B, props=props), A, B)


def _rz32(x):
    """float64 -> float32 rounded toward zero (the TMEM accumulate, R16)."""
    x = np.asarray(x, np.float64)
    f = x.astype(np.float32)
    over = np.abs(f.astype(np.float64)) > np.abs(x)
    f[over] = np.nextafter(f[over], np.float32(0))
    return f


def _split_products(a, b, variant):
    """The three exact products each K = 1 element of C is built from, in the kernel's
    MMA order: the split of R22 / 3xTF32 (p1, p2: the corrections, p3 = hi*hi)."""
    import test_tf32bf16_bound as tb
    f = np.float64
    ah, ahb, alb = (p.astype(f) for p in tb.split(a))
    bh, bhb, blb = (p.astype(f) for p in tb.split(b))
    A, Bt = np.meshgrid(np.arange(a.size), np.arange(b.size), indexing="ij")
    if variant == "tf32bf16":   # per 16-wide K step: lo'*hi', hi'*lo', hi*hi
        return alb[A] * bhb[Bt], ahb[A] * blb[Bt], ah[A] * bh[Bt]
    al = tb.rna_tf32((a - tb.rna_tf32(a)).astype(np.float32)).astype(f)   # lo = rna_tf32(x - hi)
    bl = tb.rna_tf32((b - tb.rna_tf32(b)).astype(np.float32)).astype(f)
    return al[A] * bh[Bt], ah[A] * bl[Bt], ah[A] * bh[Bt]


def test_k1_products_match_the_documented_arithmetic(props):
    """Pin of the kernel's arithmetic independent of the oracle: for K = 1 every MMA adds
    one exact product, so C follows from the split (R22 / 3xTF32), the MMA order and the
    TMEM accumulate (R16), emulated on the CPU.  Where the corrections and hi*hi share a
    sign, C is bitwise RZ(RZ(p1 + p2) + p3) (round-toward-zero adds); where they do not,
    the accumulator truncates the aligned smaller addend toward zero first, so C is that
    value or one FP32 ulp above it in magnitude (measured, R16).  A wrong operand
    offset, plane or product would be far outside either."""
    rng = np.random.default_rng(97)
    a = ((rng.random(150) * 2 - 1) * np.exp2(rng.integers(-20, 21, 150))).astype(np.float32)
    b = ((rng.random(130) * 2 - 1) * np.exp2(rng.integers(-20, 21, 130))).astype(np.float32)
    C = mm(a[:, None].copy(), b[None, :].copy(), props=props)
    p1, p2, p3 = _split_products(a, b, props["SGEMM_VARIANT"])
    model = _rz32(_rz32(p1 + p2).astype(np.float64) + p3)
    same = np.sign(p1 + p2) * np.sign(p3) >= 0
    assert np.array_equal(C[same], model[same])
    up = np.nextafter(model, np.copysign(np.float32(np.inf), model))   # one ulp away from zero
    assert np.all((C == model) | (C == up))
    assert same.mean() > 0.3 and (~same).mean() > 0.3
