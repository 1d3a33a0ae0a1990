"""GPU parity of the FP64 Ozaki-scheme task variant (K4/K5: INT8 tcgen05
slices) against the CPU oracle.

The variant is pre-selected through the Worker's PDL properties
(DGEMM_VARIANT = ozaki, OZAKI_SLICES).  Tolerance: the
same 1e-12 FP64 bar as K1, scaled by D = |A||B| (R13, R19).
Integer-valued and rank-1 inputs are represented exactly by the slices, so
those results are compared bitwise.
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
    monkeypatch.delenv("PDL_DRY_RUN", raising=False)
    monkeypatch.delenv("PDL_DGEMM_VARIANT", raising=False)
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    pdl.unload()
    yield
    pdl.unload()


def oz_matmul(A, B, tile=0, workers=1, host=False, slices=None, rounding=None):
    """Default slicing = the library's default (6 round-to-nearest slices)."""
    pdl.load(pdl.descriptor_xml(workers, "ozaki", slices, rounding))
    try:
        M, K = A.shape
        N = B.shape[1]
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


def test_variant_is_selected_from_pdl():
    pdl.load(pdl.descriptor_xml(1, "ozaki", 6))
    assert pdl.query("worker/0/DGEMM_VARIANT") == "ozaki"
    assert pdl.query("worker/0/OZAKI_SLICES") == "6"
    A = W.uniform((300, 200), np.float64, 1)
    B = W.uniform((200, 100), np.float64, 2)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    dC = torch.empty((300, 100), dtype=torch.float64, device="cuda")
    pdl.task_matmul(dA, dB, dC)
    pdl.run()
    # split A + 2 (colmax, split B) + S diagonal GEMMs
    assert pdl.query_json("stats")["launches"] == 1 + 2 + 6


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_configs_parity(name):
    c = W.CONFIGS[name]
    A, B = W.config_inputs(name, np.float64)
    check(oz_matmul(A, B, tile=c.tile), A, B)


@pytest.mark.parametrize("M,N,K", [(1, 1, 1), (3, 5, 7), (33, 31, 32), (127, 129, 128), (129, 255, 257),
                                   (257, 130, 33), (200, 17, 1000)])
def test_signed_shapes(M, N, K):
    A = W.signed((M, K), np.float64, 100 + M)
    B = W.signed((K, N), np.float64, 200 + N)
    check(oz_matmul(A, B, tile=32), A, B)
    check(oz_matmul(A, B, host=True), A, B)


def test_integer_and_rank1_bitwise():
    A = W.integers((190, 300), np.float64, 7)
    B = W.integers((300, 170), np.float64, 8)
    Cref, _ = oracle.matmul(A, B)
    assert np.array_equal(oz_matmul(A, B), Cref)
    u, v = W.rank1_factors(300, 520, 5)
    x, y = W.rank1_factors(520, 260, 6)
    expect = (int(np.dot(v, x)) * np.outer(u, y)).astype(np.float64)
    assert np.array_equal(oz_matmul(np.outer(u, v).astype(np.float64), np.outer(x, y).astype(np.float64)), expect)


def test_invariance_bitwise(monkeypatch):
    """Slices depend on whole rows of A / columns of B only, so Worker count,
    task tile and the pipelined host staging do not change a bit."""
    A = W.uniform((700, 390), np.float64, 11)
    B = W.uniform((390, 333), np.float64, 12)
    ref = oz_matmul(A, B)
    check(ref, A, B)
    for workers, tile in ((2, 64), (4, 32), (8, 0)):
        assert np.array_equal(oz_matmul(A, B, tile=tile, workers=workers), ref)
    monkeypatch.setenv("PDL_PIPELINE", "force")
    assert np.array_equal(oz_matmul(A, B, host=True), ref)


def test_k_chunks_beyond_int32_window():
    """K > 16384 is split into K chunks whose INT32 sums stay exact."""
    A = W.uniform((96, 20000), np.float64, 21)
    B = W.uniform((20000, 80), np.float64, 22)
    check(oz_matmul(A, B), A, B)


def test_wide_exponent_rows_columns():
    """Row / column scaling by powers of two: rows and columns of very
    different magnitude are each sliced relative to their own maximum."""
    A = W.signed((64, 256), np.float64, 31) * np.exp2(np.arange(64) - 32)[:, None]
    B = W.signed((256, 48), np.float64, 32) * np.exp2(3 * np.arange(48) - 60)[None, :]
    check(oz_matmul(A, B), A, B)


@pytest.mark.parametrize("slices,rounding,tol", [(6, "nearest", 1e-13), (7, "trunc", 1e-13),
                                                (5, "nearest", 1e-10), (6, "trunc", 1e-10),
                                                (8, "nearest", 1e-14)])
def test_slice_count_accuracy(slices, rounding, tol):
    """Measured error versus slice count and rounding (R19): truncation biases
    the error (U[0,1) data), round-to-nearest slices are unbiased."""
    A = W.uniform((256, 4096), np.float64, 41)
    B = W.uniform((4096, 256), np.float64, 42)
    check(oz_matmul(A, B, slices=slices, rounding=rounding), A, B, tol=tol)


def oz32_matmul(A, B, tile=0, workers=1, host=False, slices=None):
    props = {"SGEMM_VARIANT": "ozaki"}
    if slices:
        props["OZAKI_SLICES_F32"] = slices
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


@pytest.mark.parametrize("name", ["C1", "C2", "C3"])
def test_fp32_ozaki_configs(name):
    """FP32 task variant SGEMM_VARIANT = ozaki (INT8 slices of the FP32
    inputs, FP32 C) at the 1e-5 bar."""
    c = W.CONFIGS[name]
    A, B = W.config_inputs(name, np.float32)
    C = oz32_matmul(A, B, tile=c.tile)
    rows = None if c.M <= 1024 else W.sampled_rows(c.M, (), c.tile, n_random=32)
    check(C, A, B, rows=rows, tol=1e-5)


@pytest.mark.parametrize("slices,tol", [(3, 1e-5), (4, 2e-6)])
def test_fp32_ozaki_k_sweep(slices, tol, capsys):
    for K in (256, 4096, 16384):
        A = W.uniform((128, K), np.float32, 71)
        B = W.signed((K, 192), np.float32, 72)
        err = check(oz32_matmul(A, B, slices=slices), A, B, tol=tol)
        with capsys.disabled():
            print(f"\n[fp32 ozaki S={slices}] K={K} max_err={err:.3e}")


def test_fp32_ozaki_invariance_bitwise(monkeypatch):
    A = W.uniform((700, 390), np.float32, 81)
    B = W.uniform((390, 333), np.float32, 82)
    ref = oz32_matmul(A, B)
    check(ref, A, B, tol=1e-5)
    assert np.array_equal(oz32_matmul(A, B, tile=64, workers=4), ref)
    monkeypatch.setenv("PDL_PIPELINE", "force")
    assert np.array_equal(oz32_matmul(A, B, host=True), ref)


@pytest.mark.slow
def test_fp32_c4_full_size_sampled():
    c = W.CONFIGS["C4"]
    A, B = W.config_inputs("C4", np.float32)
    C = oz32_matmul(A, B, tile=c.tile)
    check(C, A, B, rows=W.sampled_rows(c.M, (), c.tile, n_random=12), tol=1e-5)


@pytest.mark.slow
@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_c5_ragged_8_workers(dt):
    """C5 ragged (10000x7000x3000, tile 128) on 8 oversubscribed Workers."""
    c = W.CONFIGS["C5"]
    npdt = np.float64 if dt == "f64" else np.float32
    A, B = W.config_inputs("C5", npdt)
    C = oz_matmul(A, B, tile=c.tile, workers=8) if dt == "f64" else oz32_matmul(A, B, tile=c.tile, workers=8)
    rows = W.sampled_rows(c.M, (1248, 2496, 3744, 5008, 6256, 7504, 8752), c.tile, n_random=24)
    check(C, A, B, rows=rows, tol=1e-12 if dt == "f64" else 1e-5)


@pytest.mark.slow
def test_c4_full_size_sampled():
    c = W.CONFIGS["C4"]
    A, B = W.config_inputs("C4", np.float64)
    C = oz_matmul(A, B, tile=c.tile)
    rows = W.sampled_rows(c.M, (), c.tile, n_random=12)
    check(C, A, B, rows=rows)
