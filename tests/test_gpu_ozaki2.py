"""GPU parity of the FP64 task variant "ozaki2" (K6/K7: Ozaki scheme II --
integer scaling, INT8 residue GEMMs on tcgen05 for pairwise-coprime moduli,
CRT reconstruction) against the CPU oracle.

Selected through the Worker's PDL properties (DGEMM_VARIANT = ozaki2,
OZAKI2_MODULI, OZAKI2_BITS).  Tolerance: the 1e-12 FP64
bar of K1 (scaled by D = |A||B|, R13).  Inputs that are integers of
at most p bits (after the power-of-two row / column scaling) are represented
exactly, and the CRT rebuilds their product exactly, so those results are
compared bitwise.
"""
import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402


@pytest.fixture(autouse=True)
def _env(monkeypatch):
    for k in ("PDL_DRY_RUN", "PDL_DGEMM_VARIANT", "PDL_OZAKI2_MODULI", "PDL_OZAKI2_BITS", "PDL_OZAKI2_GUARD",
              "PDL_OZAKI2_GUARD_TOL"):
        monkeypatch.delenv(k, raising=False)
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    pdl.unload()
    yield
    pdl.unload()


def oz2_matmul(A, B, tile=0, workers=1, host=False, moduli=None, bits=None):
    props = {"DGEMM_VARIANT": "ozaki2"}
    if moduli:
        props["OZAKI2_MODULI"] = moduli
    if bits:
        props["OZAKI2_BITS"] = bits
    pdl.load(pdl.descriptor_xml(workers, props=props))
    try:
        M, N = A.shape[0], B.shape[1]
        if host:
            C = np.full((M, N), np.nan)
            pdl.task_matmul(A, B, C, tile=tile)
            pdl.run()
            return C
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        dC = torch.full((M, N), float("nan"), dtype=torch.float64, device="cuda")
        pdl.task_matmul(dA, dB, dC, tile=tile)
        pdl.run()
        return dC.cpu().numpy()
    finally:
        pdl.unload()


def check(C, A, B, rows=None, tol=1e-12):
    Cref, D = oracle.matmul(A, B, rows=rows)
    err = oracle.scaled_error(C if rows is None else C[rows], Cref, D)
    assert np.isfinite(err).all()
    assert err.max() <= tol, f"max scaled err {err.max():.3e} > {tol:g}"
    return float(err.max())


def test_variant_selected_and_launch_count(monkeypatch):
    """13 moduli at the default 43 scaling bits for K <= 16384: A residues
    (row max, residues) + B residues (column max, residues) + 13 residue GEMMs
    (one launch each with PDL_OZ2_MERGE=1) + the CRT pass."""
    monkeypatch.setenv("PDL_OZ2_MERGE", "1")
    pdl.load(pdl.descriptor_xml(1, props={"DGEMM_VARIANT": "ozaki2"}))
    assert pdl.query("worker/0/DGEMM_VARIANT") == "ozaki2"
    A = W.uniform((300, 200), np.float64, 1)
    B = W.uniform((200, 100), np.float64, 2)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    dC = torch.empty((300, 100), dtype=torch.float64, device="cuda")
    pdl.task_matmul(dA, dB, dC)
    pdl.run()
    st = pdl.query_json("stats")
    n = st["launches"] - 5 - 3    # - the certificate GEMM, its column-term pass, K1's recompute launch
    n -= 1 if st["ozaki_guard"][0].get("certified_in_crt") else 0   # R23: the row-bound pass
    assert 11 <= n <= 13, n       # fewer moduli suffice for K = 200
    assert st["ozaki_guard"][0]["elements_recomputed"] == 0
    check(dC.cpu().numpy(), A, B)


@pytest.mark.parametrize("name", ["C1", "C2", "C3"])
def test_configs_parity(name):
    c = W.CONFIGS[name]
    A, B = W.config_inputs(name, np.float64)
    C = oz2_matmul(A, B, tile=c.tile)
    rows = None if c.M <= 1024 else W.sampled_rows(c.M, (), c.tile, n_random=32)
    check(C, A, B, rows=rows)


@pytest.mark.parametrize("M,N,K", [(1, 1, 1), (3, 5, 7), (33, 31, 32), (127, 129, 128), (129, 255, 257),
                                   (257, 130, 33), (200, 17, 1000), (300, 530, 4100)])
def test_signed_shapes(M, N, K):
    A = W.signed((M, K), np.float64, 100 + M)
    B = W.signed((K, N), np.float64, 200 + N)
    check(oz2_matmul(A, B, tile=32), A, B)
    check(oz2_matmul(A, B, host=True), A, B)


def test_integer_identity_rank1_bitwise():
    """Small integers (and their power-of-two scalings) are exact p-bit
    integers, so X = A'B' and C are exact."""
    A = W.integers((190, 300), np.float64, 7)
    B = W.integers((300, 170), np.float64, 8)
    Cref, _ = oracle.matmul(A, B)
    assert np.array_equal(oz2_matmul(A, B), Cref)
    u, v = W.rank1_factors(300, 520, 5)
    x, y = W.rank1_factors(520, 260, 6)
    expect = (int(np.dot(v, x)) * np.outer(u, y)).astype(np.float64)
    assert np.array_equal(oz2_matmul(np.outer(u, v).astype(np.float64), np.outer(x, y).astype(np.float64)), expect)
    I = W.identity(256, 256, np.float64)
    X = W.dyadic((256, 300), np.float64, 9)
    assert np.array_equal(oz2_matmul(I, X), X)


def test_zero_rows_columns_and_k0():
    A = W.uniform((130, 90), np.float64, 3)
    B = W.uniform((90, 70), np.float64, 4)
    A[5] = 0.0
    B[:, 7] = 0.0
    C = oz2_matmul(A, B)
    assert np.all(C[5] == 0.0) and np.all(C[:, 7] == 0.0)
    check(C, A, B)


def test_invariance_bitwise(monkeypatch):
    """Scaling exponents come from whole rows of A / columns of B and the
    CRT is exact, so Worker count, tile and pipelined staging change no bit."""
    A = W.uniform((700, 390), np.float64, 11)
    B = W.uniform((390, 333), np.float64, 12)
    ref = oz2_matmul(A, B)
    check(ref, A, B)
    for workers, tile in ((2, 64), (4, 32), (8, 0)):
        assert np.array_equal(oz2_matmul(A, B, tile=tile, workers=workers), ref)
    monkeypatch.setenv("PDL_PIPELINE", "force")
    assert np.array_equal(oz2_matmul(A, B, host=True), ref)


def test_gemm_shapes_and_crt_passes_bitwise(monkeypatch):
    """The residue GEMMs are exact INT32 sums and the CRT is exact, so the K6
    kernel shape (persistent 256 x 512 -- the default for this size, >= 148
    cluster tiles --, one cluster per tile, 256 x 256, two CTA pairs per SM),
    the moduli per persistent launch (default 6 + 7 here: 2.2 rounds of tiles
    per modulus; 1, 5 and all 13 forced),
    and the serpentine-K / cache-hint knobs change no bit; ragged edges in both
    dimensions.  The 128-bit integer CRT pass rounds X twice (high and low words),
    the FP64 pass once, so those agree to 2 ulps."""
    A = W.uniform((5000, 1100), np.float64, 21) - 0.5
    B = W.uniform((1100, 3999), np.float64, 22)
    ref = oz2_matmul(A, B)
    rows = [0, 1, 255, 256, 4095, 4999] + list(np.random.default_rng(3).integers(0, 5000, 24))
    check(ref, A, B, rows=rows)
    for env in ({"PDL_OZ2_PERSIST": "0"}, {"PDL_OZ_SHAPE": "256"}, {"PDL_OZ_SHAPE": "256x2"},
                {"PDL_OZ2_HINTS": "7"}, {"PDL_OZ2_MERGE": "1"}, {"PDL_OZ2_MERGE": "5"},
                {"PDL_OZ2_MERGE": "13"}):
        with monkeypatch.context() as mp:
            for k, v in env.items():
                mp.setenv(k, v)
            assert np.array_equal(oz2_matmul(A, B), ref), env
    monkeypatch.setenv("PDL_OZ2_CRT", "int")
    Ci = oz2_matmul(A, B)
    assert np.all(np.abs(Ci - ref) <= 2 * np.spacing(np.abs(ref)))


def test_k_chunks_beyond_int32_window():
    """K > 65536 is split into K chunks (each CRT-exact), summed in FP64."""
    A = W.uniform((64, 70000), np.float64, 21)
    B = W.uniform((70000, 48), np.float64, 22)
    check(oz2_matmul(A, B), A, B)


def test_wide_exponent_rows_columns():
    A = W.signed((64, 256), np.float64, 31) * np.exp2(np.arange(64) - 32)[:, None]
    B = W.signed((256, 48), np.float64, 32) * np.exp2(3 * np.arange(48) - 60)[None, :]
    check(oz2_matmul(A, B), A, B)


def test_scaling_bits_above_50_residue_fallback():
    """14 moduli at K <= 128 give p = 51 > 50: |A'| may reach 2^51, beyond the
    one-DFMA residue path's exactness bound, so K7 takes the four-op residue path
    with fix-ups (k_ozaki2.cu res8); both sides of the bound stay within the bar."""
    import json
    pdl.load(pdl.descriptor_xml(1))
    try:
        assert json.loads(pdl.query("ozaki2_plan/100/43/14"))["p"] == 51
        assert json.loads(pdl.query("ozaki2_plan/300/43/14"))["p"] == 50
    finally:
        pdl.unload()
    for K in (100, 300):
        A = W.signed((96, K), np.float64, 51) * np.exp2(np.arange(96) % 7 - 3)[:, None]
        B = W.uniform((K, 80), np.float64, 52)
        check(oz2_matmul(A, B, moduli=14), A, B, tol=1e-15)


@pytest.mark.parametrize("moduli,tol", [(13, 1e-13), (14, 1e-14), (11, 1e-9)])
def test_moduli_count_accuracy(moduli, tol, monkeypatch):
    """Fewer moduli force fewer scaling bits p (|X| <= K 2^(2p) < M/2): the
    raw accuracy of the residue arithmetic, certificate off (with it on, 11
    moduli send every element to K1)."""
    monkeypatch.setenv("PDL_OZAKI2_GUARD", "off")
    A = W.uniform((256, 4096), np.float64, 41)
    B = W.signed((4096, 256), np.float64, 42)
    check(oz2_matmul(A, B, moduli=moduli), A, B, tol=tol)


@pytest.mark.slow
def test_c4_full_size_sampled():
    c = W.CONFIGS["C4"]
    A, B = W.config_inputs("C4", np.float64)
    C = oz2_matmul(A, B, tile=c.tile)
    check(C, A, B, rows=W.sampled_rows(c.M, (), c.tile, n_random=12))


@pytest.mark.slow
def test_c5_ragged_8_workers():
    c = W.CONFIGS["C5"]
    A, B = W.config_inputs("C5", np.float64)
    C = oz2_matmul(A, B, tile=c.tile, workers=8)
    rows = W.sampled_rows(c.M, (1248, 2496, 3744, 5008, 6256, 7504, 8752), c.tile, n_random=24)
    check(C, A, B, rows=rows)


def test_fp32_ozaki2_is_unsupported():
    pdl.load(pdl.descriptor_xml(1, props={"SGEMM_VARIANT": "ozaki2"}))
    A = torch.rand((64, 64), device="cuda")
    C = torch.empty((64, 64), device="cuda")
    pdl.task_matmul(A, A, C)
    with pytest.raises(pdl.PDLError) as e:
        pdl.run()
    assert e.value.code == pdl.PDL_EUNSUPPORTED


def test_k0_and_tiny():
    dA = torch.empty((40, 0), dtype=torch.float64, device="cuda")
    dB = torch.empty((0, 30), dtype=torch.float64, device="cuda")
    dC = torch.full((40, 30), float("nan"), dtype=torch.float64, device="cuda")
    pdl.load(pdl.descriptor_xml(1, props={"DGEMM_VARIANT": "ozaki2"}))
    pdl.task_matmul(dA, dB, dC, M=40, N=30, K=0)
    pdl.run()
    assert torch.count_nonzero(dC).item() == 0
    pdl.unload()
    A = W.signed((1, 1), np.float64, 3)
    B = W.signed((1, 1), np.float64, 4)
    check(oz2_matmul(A, B), A, B)           # 53-bit inputs, p-bit scaling: within the bar
    A, B = np.array([[3.0]]), np.array([[-0.625]])
    assert np.array_equal(oz2_matmul(A, B), A @ B)     # short mantissas: exact


# ---- the certificate (R21) ----------------------------------------

def oz2_run(A, B, guard=True, workers=1, tile=0, variant="ozaki2"):
    """C and the certificate stats of one run (device-resident operands)."""
    props = {"DGEMM_VARIANT": variant}
    if variant == "ozaki2" and not guard:
        props["OZAKI2_GUARD"] = "off"
    pdl.load(pdl.descriptor_xml(workers, props=props))
    try:
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        dC = torch.full((A.shape[0], B.shape[1]), float("nan"), dtype=torch.float64, device="cuda")
        pdl.task_matmul(dA, dB, dC, tile=tile)
        pdl.run()
        st = pdl.query_json("stats")
        return dC.cpu().numpy(), st.get("ozaki_guard", [])
    finally:
        pdl.unload()


def recomputed(g):
    return sum(w["elements_recomputed"] for w in g)


def adversarial(kind, seed):
    rng = np.random.default_rng(seed)
    if kind == "huge_times_zero":
        # [2^60, 1] x [0, 1]^T: the 1 is below Ozaki II's 2^-43 row resolution
        A = W.uniform((300, 200), np.float64, seed)
        B = W.uniform((200, 260), np.float64, seed + 1)
        A[7, :2] = [2.0 ** 60, 1.0]
        A[7, 2:] = 0.0
        B[:2, 11] = [0.0, 1.0]
        A[150, 3] = 2.0 ** 60          # one huge element meeting zeros of B
        B[3, :] = 0.0
        return A, B
    if kind == "in_row_spread":
        # every element scaled by 2^u, u uniform in [-60, 60]: rows and columns
        # spanning 120 binades
        A = W.signed((256, 384), np.float64, seed) * np.exp2(rng.integers(-60, 61, (256, 384)))
        B = W.signed((384, 200), np.float64, seed + 1) * np.exp2(rng.integers(-60, 61, (384, 200)))
        return A, B
    if kind.startswith("cancel_k"):
        # small K with signed entries and exact cancellation partners: D_ij stays
        # ~|a||b| while C_ij is tiny, and D_ij can be far below K max|a_i| max|b_j|
        K = int(kind[8:])
        A = W.signed((512, K), np.float64, seed) * np.exp2(rng.integers(-20, 21, (512, K)))
        B = W.signed((K, 384), np.float64, seed + 1) * np.exp2(rng.integers(-20, 21, (K, 384)))
        if K >= 2:
            A[:, 1] = -A[:, 0] * (1 + 2.0 ** -30)
            B[1, :] = B[0, :]
        return A, B
    raise ValueError(kind)


KINDS = ["huge_times_zero", "in_row_spread"] + [f"cancel_k{k}" for k in (2, 3, 4, 8, 16)]


@pytest.mark.parametrize("kind", KINDS)
def test_certificate_holds_on_adversarial_inputs(kind):
    """Seeded adversarial inputs at the plain 1e-12 componentwise bar through
    DGEMM_VARIANT=ozaki2: the elements whose certified bound exceeds tau D_ij
    are recomputed by K1; the others are certified."""
    A, B = adversarial(kind, 7)
    C, g = oz2_run(A, B)
    check(C, A, B)
    if kind in ("huge_times_zero", "in_row_spread"):
        assert recomputed(g) > 0, "these inputs need the K1 recompute"
    if kind == "huge_times_zero":
        assert C[7, 11] == 1.0


@pytest.mark.parametrize("kind", ["huge_times_zero", "in_row_spread"])
def test_without_the_certificate_the_bar_fails(kind):
    """Negative control: the same inputs with OZAKI2_GUARD=off break the 1e-12
    bar, so the certificate is what holds it."""
    A, B = adversarial(kind, 7)
    C, _ = oz2_run(A, B, guard=False)
    Cref, D = oracle.matmul(A, B)
    assert oracle.scaled_error(C, Cref, D).max() > 1e-12


def test_recomputed_elements_are_k1_bits_and_the_rest_ozaki_bits():
    """Each element is either certified (bitwise the unguarded Ozaki-II value)
    or recomputed (bitwise the K1 value) -- decided from its own row / column
    sums and certificate product only."""
    A, B = adversarial("in_row_spread", 11)
    C, g = oz2_run(A, B)
    C_off, _ = oz2_run(A, B, guard=False)
    C_k1, _ = oz2_run(A, B, variant="dmma")
    same_oz = C == C_off
    same_k1 = C == C_k1
    assert np.all(same_oz | same_k1)
    assert recomputed(g) >= np.count_nonzero(~same_oz)


def test_certificate_invariant_under_workers_and_tiles():
    """The recompute set is per element, so Worker count and task tile change
    no bit of the guarded result either (R14)."""
    A, B = adversarial("cancel_k4", 13)
    ref, _ = oz2_run(A, B)
    for workers, tile in ((2, 64), (4, 32), (8, 0)):
        C, _ = oz2_run(A, B, workers=workers, tile=tile)
        assert np.array_equal(C, ref), (workers, tile)


@pytest.mark.parametrize("name", ["C2", "C3"])
def test_certificate_passes_benign_workloads(name):
    """U[0,1) and U[-1,1) workloads of the configs are certified everywhere:
    no element goes to K1 (the guard costs one INT8 GEMM, no recompute)."""
    A, B = W.config_inputs(name, np.float64)
    C, g = oz2_run(A, B)
    assert recomputed(g) == 0
    assert sum(w["tiles_checked"] for w in g) == -(-A.shape[0] // 128) * -(-B.shape[1] // 128)
    Cs, gs = oz2_run(2 * A - 1, 2 * B - 1)
    assert recomputed(gs) == 0


# ---- the certificate of sign-uniform rows and columns (R23) ---------

def oz2_run_env(A, B, monkeypatch, uniform=True, workers=1, tile=0, host=False):
    if uniform:
        monkeypatch.delenv("PDL_OZ2_CERT_UNIFORM", raising=False)
    else:
        monkeypatch.setenv("PDL_OZ2_CERT_UNIFORM", "0")
    pdl.load(pdl.descriptor_xml(workers, props={"DGEMM_VARIANT": "ozaki2"}))
    try:
        if host:
            C = np.full((A.shape[0], B.shape[1]), np.nan)
            pdl.task_matmul(A, B, C, tile=tile)
            pdl.run()
        else:
            dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
            dC = torch.full((A.shape[0], B.shape[1]), float("nan"), dtype=torch.float64, device="cuda")
            pdl.task_matmul(dA, dB, dC, tile=tile)
            pdl.run()
            C = dC.cpu().numpy()
        return C, pdl.query_json("stats").get("ozaki_guard", [])
    finally:
        pdl.unload()


def gsum(g, key):
    return sum(w.get(key, 0) for w in g)


def test_uniform_operands_skip_the_certificate_gemm(monkeypatch):
    """U[0,1) operands: every row and column is sign-uniform, so D = |C| and the CRT
    pass certifies every element; the lower-bound GEMM is skipped.  Benign data is
    certified either way, so C is bitwise the GEMM-certificate result."""
    A, B = W.config_inputs("C3", np.float64)
    C, g = oz2_run_env(A, B, monkeypatch)
    check(C, A, B, rows=np.arange(0, A.shape[0], 37))
    assert gsum(g, "certified_in_crt") >= 1 and gsum(g, "certificate_gemms_skipped") >= 1
    assert recomputed(g) == 0
    C0, g0 = oz2_run_env(A, B, monkeypatch, uniform=False)
    assert gsum(g0, "certificate_gemms_skipped") == 0 and gsum(g0, "certified_in_crt") == 0
    assert np.array_equal(C, C0)
    # all-negative rows times positive columns are sign-uniform too
    C1, g1 = oz2_run_env(-A, B, monkeypatch)
    assert gsum(g1, "certificate_gemms_skipped") >= 1
    assert np.array_equal(C1, -C)


def positive_adversarial(seed):
    """Non-negative operands (every row and column sign-uniform) that Ozaki II's
    p-bit scaling cannot represent: in-row spread over 2^+-60 and [2^60, 1] x [0, 1]^T."""
    rng = np.random.default_rng(seed)
    A = W.uniform((256, 384), np.float64, seed) * np.exp2(rng.integers(-60, 61, (256, 384)))
    B = W.uniform((384, 200), np.float64, seed + 1) * np.exp2(rng.integers(-60, 61, (384, 200)))
    A[7, :2] = [2.0 ** 60, 1.0]
    A[7, 2:] = 0.0
    B[:2, 11] = [0.0, 1.0]
    return A, B


def test_uniform_certificate_flags_what_it_cannot_certify(monkeypatch):
    """The CRT-pass certificate is a certificate: on non-negative adversarial operands
    it sends the elements it cannot certify to K1 and the 1e-12 bar holds; without any
    certificate (OZAKI2_GUARD=off) the same inputs break the bar."""
    A, B = positive_adversarial(21)
    C, g = oz2_run_env(A, B, monkeypatch)
    check(C, A, B)
    assert gsum(g, "certificate_gemms_skipped") >= 1
    assert recomputed(g) > 0
    assert C[7, 11] == 1.0
    C_off, _ = oz2_run(A, B, guard=False)
    Cref, D = oracle.matmul(A, B)
    assert oracle.scaled_error(C_off, Cref, D).max() > 1e-12


def mixed_adversarial(seed):
    """Some rows / columns mix signs, the rest are uniform, with adversarial entries in
    both kinds: each element is certified by its own kind's certificate."""
    A, B = positive_adversarial(seed)
    rng = np.random.default_rng(seed + 7)
    mr = rng.choice(A.shape[0], 60, replace=False)
    A[mr] *= np.where(rng.random((60, A.shape[1])) < 0.5, -1.0, 1.0)
    mc = rng.choice(B.shape[1], 50, replace=False)
    B[:, mc] *= np.where(rng.random((B.shape[0], 50)) < 0.5, -1.0, 1.0)
    A[7, 2:] = 0.0     # keep row 7 the [2^60, 1] case (uniform)
    return A, B


def test_mixed_sign_operands_use_both_certificates(monkeypatch):
    A, B = mixed_adversarial(31)
    C, g = oz2_run_env(A, B, monkeypatch)
    check(C, A, B)
    assert gsum(g, "certificate_gemms_skipped") == 0 and gsum(g, "certified_in_crt") >= 1
    assert recomputed(g) > 0
    C0, _ = oz2_run_env(A, B, monkeypatch, uniform=False)
    check(C0, A, B)


def test_uniform_certificate_invariant_under_workers_tiles_and_staging(monkeypatch):
    """R14: the choice between the two certificates is per element (its row's and
    column's signs), never per launch, so Worker count, task tile and the host-staged
    band x panel cut change no bit -- even where one Worker's rectangle is all
    sign-uniform and another's is not."""
    A, B = mixed_adversarial(41)
    ref, _ = oz2_run_env(A, B, monkeypatch)
    check(ref, A, B)
    for workers, tile in ((2, 64), (4, 32), (8, 0)):
        C, _ = oz2_run_env(A, B, monkeypatch, workers=workers, tile=tile)
        assert np.array_equal(C, ref), (workers, tile)
    monkeypatch.setenv("PDL_PIPELINE", "force")
    C, _ = oz2_run_env(A, B, monkeypatch, host=True, tile=64)
    assert np.array_equal(C, ref)
