"""The Worker<->Worker exchange behind the C ABI (PAPER.md
SS IV-C step 3, L1336-1341: transfer paths derived from the descriptor's
interconnects).  One process drives G Workers of the shipped B200 descriptors
(NVLink Interconnect among the replicated Workers); on this 1-GPU box they are
oversubscribed onto cuda:0, so the peer copies run device-to-device through the
same code path they take over NVLink.

Checked: host operands cross the Master->Worker interconnect exactly once
((M K + K N) s bytes), the Workers receive the rest of their panels from each
other (the a5 formula), C is gathered once (M N s), and C is bitwise the
single-Worker result (R14) -- for every task variant and ragged shapes."""
import os
import subprocess

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _env(monkeypatch):
    monkeypatch.delenv("PDL_DRY_RUN", raising=False)
    monkeypatch.delenv("PDL_EXCHANGE", raising=False)
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    pdl.unload()
    yield
    pdl.unload()


def host_run(A, B, G, tile, props=None):
    pdl.load(pdl.descriptor_xml(G, props=props) if props else pdl.descriptor_path(G))
    try:
        C = np.full((A.shape[0], B.shape[1]), np.nan, dtype=A.dtype)
        pdl.task_matmul(A, B, C, tile=tile)
        pdl.run()
        stats = pdl.query_json("stats")
        plans = [pdl.plan(A.shape[0], B.shape[1], A.shape[1], tile, worker=w) for w in range(G)]
        return C, stats, plans
    finally:
        pdl.unload()


def expected_w2w(plans, K, es):
    """a5: each Worker receives the other Gc - 1 chunks of its A row-panel and
    the other Gr - 1 chunks of its B column-panel (ragged chunks as planned)."""
    tot = 0
    for p in plans:
        rows, cols = p["row1"] - p["row0"], p["col1"] - p["col0"]
        for j in range(p["Gc"]):
            if j != p["c"]:
                lo = min(j * p["qa"], rows)
                tot += (min(lo + p["qa"], rows) - lo) * K * es
        for r in range(p["Gr"]):
            if r != p["r"]:
                lo = min(r * p["qb"], K)
                tot += (min(lo + p["qb"], K) - lo) * cols * es
    return tot


CASES = [
    # (G, dtype, M, N, K, tile, variant)
    (2, np.float64, 1000, 700, 300, 128, None),
    (4, np.float64, 1024, 1024, 512, 128, None),
    (8, np.float64, 1000, 700, 300, 64, None),
    (8, np.float32, 1000, 700, 300, 64, None),
    (8, np.float64, 777, 513, 1000, 128, "ozaki2"),
    (4, np.float64, 1500, 1100, 260, 128, "ozaki2"),
]


@pytest.mark.parametrize("G,dt,M,N,K,tile,variant", CASES)
def test_exchange_bytes_and_bitwise(G, dt, M, N, K, tile, variant):
    rng = np.random.default_rng(G * 1000 + K)
    A = rng.uniform(-1, 1, (M, K)).astype(dt)
    B = rng.uniform(-1, 1, (K, N)).astype(dt)
    props = None
    if variant:
        props = {"DGEMM_VARIANT" if dt == np.float64 else "SGEMM_VARIANT": variant}
    C1, s1, _ = host_run(A, B, 1, tile, props)
    CG, sG, plans = host_run(A, B, G, tile, props)
    es = np.dtype(dt).itemsize
    tr = sG["transfers"]
    assert tr["exchange_tasks"] == 1
    assert tr["master_to_worker"] == (M * K + K * N) * es          # each operand byte crosses PCIe once
    assert tr["worker_to_master"] == M * N * es                    # C gathered once
    assert tr["worker_to_worker"] == expected_w2w(plans, K, es) > 0
    assert tr["master_worker_ic"] == "PCIe" and tr["worker_worker_ic"] == "NVLink"
    assert s1["transfers"]["worker_to_worker"] == 0
    assert np.array_equal(C1, CG), "C differs from the single-Worker result"
    rows = np.unique(np.r_[0, M - 1, [p["row0"] for p in plans], [p["row1"] - 1 for p in plans],
                          np.arange(0, M, 61)])
    Cref, D = oracle.matmul(A, B, rows=rows)
    tol = 1e-12 if dt == np.float64 else 1e-5
    assert (oracle.scaled_error(CG[rows], Cref, D) <= tol).all()


def test_exchange_off_stages_whole_panels(monkeypatch):
    """PDL_EXCHANGE=0 (or a descriptor without a Worker<->Worker interconnect):
    every Worker stages its whole panels through the Master's memory region --
    (Gc M K + Gr K N) s over PCIe -- and C is the same bits."""
    A, B = W.config_inputs("C1", np.float64)
    A = np.ascontiguousarray(np.tile(A, (4, 3)))
    B = np.ascontiguousarray(np.tile(B, (3, 5)))
    C_x, s_x, plans = host_run(A, B, 8, 32)
    monkeypatch.setenv("PDL_EXCHANGE", "0")
    C_h, s_h, _ = host_run(A, B, 8, 32)
    M, K = A.shape
    N = B.shape[1]
    Gr, Gc = plans[0]["Gr"], plans[0]["Gc"]
    assert s_h["transfers"]["exchange_tasks"] == 0 and s_h["transfers"]["worker_to_worker"] == 0
    assert s_h["transfers"]["master_to_worker"] == (Gc * M * K + Gr * K * N) * 8
    assert s_x["transfers"]["master_to_worker"] == (M * K + K * N) * 8
    assert np.array_equal(C_x, C_h)


def test_exchange_repeated_runs_and_async():
    """Back-to-back asynchronous runs reuse the panel buffers: the second run's
    unique-chunk copies wait for the first run's readers."""
    rng = np.random.default_rng(3)
    M, N, K = 900, 650, 400
    pdl.load(pdl.descriptor_path(8))
    try:
        outs = []
        for seed in (1, 2, 3):
            A = np.random.default_rng(seed).uniform(0, 1, (M, K))
            B = np.random.default_rng(seed + 10).uniform(0, 1, (K, N))
            C = np.full((M, N), np.nan)
            pdl.task_matmul(A, B, C, tile=64)
            pdl.run_async()
            outs.append((A, B, C))
        pdl.sync()
        for A, B, C in outs:
            rows = rng.integers(0, M, 20)
            Cref, D = oracle.matmul(A, B, rows=rows)
            assert (oracle.scaled_error(C[rows], Cref, D) <= 1e-12).all()
    finally:
        pdl.unload()


def test_sync_timeout_reports_the_exchange(monkeypatch):
    """PDL_SYNC_TIMEOUT_MS bounds pdl_sync; a run that completes in time is OK."""
    monkeypatch.setenv("PDL_SYNC_TIMEOUT_MS", "60000")
    A, B = W.config_inputs("C2", np.float64)
    C, s, _ = host_run(A, B, 4, 128)
    assert s["transfers"]["exchange_tasks"] == 1
    rows = np.arange(0, 1024, 101)
    Cref, D = oracle.matmul(A, B, rows=rows)
    assert (oracle.scaled_error(C[rows], Cref, D) <= 1e-12).all()


def test_c_example_eight_workers():
    """The C-only example through the C ABI with the 8-Worker descriptor: the
    exchange runs behind pdl_run with no Python on the path."""
    r = subprocess.run(["make", "-C", ROOT, "examples"], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    env = dict(os.environ, PDL_ALLOW_OVERSUBSCRIBE="1")
    r = subprocess.run([os.path.join(ROOT, "examples", "dgemm_c_abi"),
                        os.path.join(ROOT, "paper_conf_ipps_sandrieserbp11_b200", "descriptors", "b200_x8.xml"),
                        "1536"], capture_output=True, text=True, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "worker_to_worker" in r.stdout
