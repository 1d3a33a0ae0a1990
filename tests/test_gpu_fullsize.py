"""Exact pins at the full sizes of the paper-shaped workloads (SURVEY.md SS8(c)
P4, P5, P7; the paper's 8192^2 / 16384^2 DGEMM scale), in
the launch configuration bench.py times.

* P4 rank-1 closed form at C4 (16384^3) and C5 (10000 x 7000 x 3000): A = u v^T,
  B = x y^T with integer factors in [-4, 4]; C = (v.x) u y^T exactly (|C| <= 2^22,
  exact in FP32 and TF32 too).  Compared bitwise on EVERY element against the
  closed form computed in int64 on the host -- no oracle run, no GPU arithmetic
  in the expected value -- for K1 (FP64 DMMA), K2 (FP32: the default tf32bf16 and
  3xTF32) and Ozaki II.
* P5 integer matrices in {-8..8} at C4: every partial sum is an integer below
  2^20, so C equals the oracle bitwise on 256 sampled rows (all columns).
* P7 at C4 on the 8-Worker descriptor (oversubscribed on this GPU): C is
  bitwise the single-Worker C, and every Worker-boundary row +-1 matches the
  oracle within 1e-12.
"""
import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
torch = pytest.importorskip("torch")
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402


@pytest.fixture(autouse=True)
def _env(monkeypatch):
    for k in ("PDL_DRY_RUN", "PDL_DGEMM_VARIANT", "PDL_SGEMM_VARIANT", "PDL_OZAKI2_GUARD"):
        monkeypatch.delenv(k, raising=False)
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    pdl.unload()
    yield
    pdl.unload()
    torch.cuda.empty_cache()


def run(A, B, dt, tile, workers=1, variant=None):
    """One task on device-resident operands through the C ABI; C back on the host."""
    props = None
    if variant:
        props = {("SGEMM_VARIANT" if dt == np.float32 else "DGEMM_VARIANT"): variant}
    pdl.load(pdl.descriptor_xml(workers, props=props) if props else pdl.descriptor_path(workers))
    try:
        dA = torch.from_numpy(A).cuda()
        dB = torch.from_numpy(B).cuda()
        dC = torch.full((A.shape[0], B.shape[1]), float("nan"), dtype=dA.dtype, device="cuda")
        pdl.task_matmul(dA, dB, dC, tile=tile)
        pdl.run()
        del dA, dB
        return dC.cpu().numpy()
    finally:
        pdl.unload()


def rank1(name, dt):
    c = W.CONFIGS[name]
    u, v = W.rank1_factors(c.M, c.K, 40 + c.cid)
    x, y = W.rank1_factors(c.K, c.N, 50 + c.cid)
    A = np.outer(u, v).astype(dt)
    B = np.outer(x, y).astype(dt)
    s = int(np.dot(v, x))                       # exact int64
    expect = (s * np.outer(u, y)).astype(dt)    # int64, |.| <= 2^22: exact in dt
    return A, B, expect


@pytest.mark.parametrize("name", ["C4", "C5"])
@pytest.mark.parametrize("dt,variant", [(np.float64, None), (np.float32, None), (np.float32, "3xtf32"),
                                        (np.float64, "ozaki2")])
def test_rank1_closed_form_every_element(name, dt, variant):
    c = W.CONFIGS[name]
    A, B, expect = rank1(name, dt)
    workers = 8 if name == "C5" else 1
    C = run(A, B, dt, c.tile, workers=workers, variant=variant)
    bad = np.count_nonzero(C != expect)
    assert bad == 0, f"{bad} of {C.size} elements differ from the closed form"


@pytest.mark.parametrize("dt,variant", [(np.float64, None), (np.float32, None), (np.float32, "3xtf32"),
                                        (np.float64, "ozaki2")])
def test_integer_matrices_c4_bitwise_sampled(dt, variant):
    c = W.CONFIGS["C4"]
    A, B = W.config_inputs("C4", dt, dist="integers")
    C = run(A, B, dt, c.tile, variant=variant)
    rows = W.sampled_rows(c.M, (), c.tile, n_random=262)
    assert len(rows) >= 256
    Cref, _ = oracle.matmul(A, B, rows=rows)
    assert np.array_equal(C[rows].astype(np.float64), Cref)


def test_c4_eight_workers_bitwise_and_boundary_rows():
    c = W.CONFIGS["C4"]
    A, B = W.config_inputs("C4", np.float64)
    C1 = run(A, B, np.float64, c.tile, workers=1)
    C8 = run(A, B, np.float64, c.tile, workers=8)
    assert np.array_equal(C1, C8)
    pdl.load(pdl.descriptor_path(8))
    try:
        plans = [pdl.plan(c.M, c.N, c.K, c.tile, worker=w) for w in range(8)]
    finally:
        pdl.unload()
    bounds = sorted({p["row0"] for p in plans} | {p["row1"] for p in plans})
    rows = W.sampled_rows(c.M, bounds, c.tile, n_random=24)
    Cref, D = oracle.matmul(A, B, rows=rows)
    err = oracle.scaled_error(C8[rows], Cref, D)
    assert err.max() <= 1e-12, err.max()
    # every Worker-boundary column +-1 too (all rows of the sample)
    cols = sorted({p["col0"] for p in plans} | {p["col1"] for p in plans})
    cset = sorted({j + d for j in cols for d in (-1, 0, 1) if 0 <= j + d < c.N})
    assert (err[:, cset] <= 1e-12).all()
