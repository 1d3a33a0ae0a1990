"""One-process-per-Worker path on the GPU: 2 and 4 ranks under torchrun run
the public API runtime.distributed_matmul (BLOCK plan from libpdl, chunk
staging, all-gather exchange, local tile kernel, gather of C) and check their
rectangles against the oracle.  With a single B200 the ranks share it and the
exchange runs over gloo (NCCL forbids two ranks on one GPU); on a multi-GPU
box the same script runs over NCCL.
"""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(world, *args, env_extra=None):
    torch = pytest.importorskip("torch")
    backend = "nccl" if torch.cuda.device_count() >= world else "gloo"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={_port()}", os.path.join(ROOT, "tests", "dist_check.py"),
           *[str(a) for a in args[:5]], backend, *[str(a) for a in args[5:]]]
    env = dict(os.environ, PDL_ALLOW_OVERSUBSCRIBE="1", **(env_extra or {}))
    env.pop("PDL_DRY_RUN", None)
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    errs = [ln for ln in r.stderr.splitlines() if "Error" in ln or "error" in ln or "dist_check" in ln]
    assert r.returncode == 0, r.stdout[-3000:] + "\n".join(errs[:40]) + r.stderr[-1500:]
    assert "ok=True" in r.stdout


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_distributed_matmul(world, dt):
    _run(world, dt, 1000, 700, 300, 128)


@pytest.mark.parametrize("overlap", ["0", "1"])
def test_distributed_ragged_8(overlap):
    """Both A-exchange policies: one launch after the whole exchange (the default
    at this size) and the chunked overlap (PDL_OVERLAP_A=1)."""
    _run(8, "f64", 1000, 700, 300, 64, env_extra={"PDL_OVERLAP_A": overlap})


def test_distributed_ozaki2_4():
    _run(4, "f64", 777, 513, 1000, 128, "ozaki2")


@pytest.mark.parametrize("G,dt,variant", [(4, "f64", None), (8, "f64", None), (8, "f32", None),
                                          (8, "f64", "ozaki2"), (4, "f64", "ozaki2")])
def test_concurrent_chunk_groups_bitwise(G, dt, variant, monkeypatch):
    """runtime.compute_groups with the later chunk groups on side streams, each
    task in its own libpdl scratch slot (PDL_TASK_SLOT) and reusing the B panel
    prepared on the Worker stream, gives bitwise the serial launches' C for
    every Worker position of a G-Worker plan and every task variant, and sampled
    rows match the oracle."""
    torch = pytest.importorskip("torch")
    import numpy as np

    sys.path.insert(0, ROOT)
    import oracle
    from paper_conf_ipps_sandrieserbp11_b200 import pdl, runtime

    if variant:
        monkeypatch.setenv("PDL_DGEMM_VARIANT" if dt == "f64" else "PDL_SGEMM_VARIANT", variant)
    M, N, K, tile = 1500, 1100, 260, 128
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    monkeypatch.setenv("PDL_DRY_RUN", "1")
    pdl.load(pdl.descriptor_path(G))
    try:
        wps = [runtime.worker_plan(M, N, K, tile, r) for r in range(G)]
    finally:
        pdl.unload()
        monkeypatch.delenv("PDL_DRY_RUN")
    npdt, tdt = (np.float64, torch.float64) if dt == "f64" else (np.float32, torch.float32)
    rng = np.random.default_rng(5)
    A = rng.uniform(-1, 1, (M, K)).astype(npdt)
    B = rng.uniform(-1, 1, (K, N)).astype(npdt)
    dev = torch.device("cuda", 0)
    tol = 1e-12 if dt == "f64" else 1e-5
    pdl.load(pdl.descriptor_path(1))
    try:
        assert pdl.query("concurrent_tasks/" + dt) == "yes"
        for wp in wps:
            bufs = runtime.PanelBuffers(wp, tdt, dev)
            bufs.A.zero_()
            bufs.A[: wp.rows].copy_(torch.from_numpy(A[wp.row0: wp.row1]))
            bufs.B[: wp.K].copy_(torch.from_numpy(B[:, wp.col0: wp.col1]))
            Bp = bufs.B[: wp.K]
            assert runtime.tasks_may_overlap(bufs.A, Bp)
            out = []
            for conc in (False, True, True):
                C = torch.full((wp.rows, wp.cols), float("nan"), dtype=tdt, device=dev)
                pdl.set_stream(torch.cuda.current_stream())
                runtime.compute_groups(wp, bufs, Bp, runtime.chunk_task(C, wp, tile), {}, conc)
                pdl.sync()
                torch.cuda.synchronize()
                out.append(C.cpu().numpy())
            assert np.array_equal(out[0], out[1]) and np.array_equal(out[0], out[2]), (wp.r, wp.c)
            rows = np.arange(0, wp.rows, 97)
            Cref, D = oracle.matmul(A[wp.row0: wp.row1][rows], B[:, wp.col0: wp.col1])
            assert (oracle.scaled_error(out[1][rows], Cref, D) <= tol).all()
    finally:
        pdl.unload()


def _run_rc(world, *args, env_extra=None):
    torch = pytest.importorskip("torch")
    backend = "nccl" if torch.cuda.device_count() >= world else "gloo"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={_port()}", os.path.join(ROOT, "tests", "dist_check.py"),
           *[str(a) for a in args[:5]], backend, *[str(a) for a in args[5:]]]
    env = dict(os.environ, PDL_ALLOW_OVERSUBSCRIBE="1", **(env_extra or {}))
    env.pop("PDL_DRY_RUN", None)
    return subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)


@pytest.mark.parametrize("world,dt", [(4, "f64"), (8, "f64"), (8, "f32")])
def test_late_chunks_are_waited_for(world, dt):
    """Every A chunk and B chunk lands 3 ms late on the comm stream (a spin kernel
    before the landing copy) into NaN-poisoned panel buffers, while the host runs
    ahead (the collectives have NCCL's stream semantics): C is still correct, so
    every compute launch of compute_groups waits for its own chunks."""
    _run(world, dt, 1000, 700, 300, 64,
         env_extra={"PDL_TEST_EXCHANGE_DELAY_US": "3000", "PDL_OVERLAP_A": "1"})


@pytest.mark.parametrize("world", [4, 8])
def test_ozaki2_prepared_exchange_with_late_raw_rows(world):
    """Ozaki-II exchanges prepared chunks (residues + row scales + certificate
    sums) and, after them, the raw chunks its certificate's K1 recompute reads;
    with every landing 3 ms late and adversarial rows that force the recompute,
    C is still right: the recompute waits for its raw rows (raw_ready event)."""
    _run(world, "f64", 1000, 700, 300, 64, "ozaki2",
         env_extra={"PDL_TEST_EXCHANGE_DELAY_US": "3000", "PDL_OVERLAP_A": "1", "DIST_CHECK_ADVERSARIAL": "1"})


def test_a_missing_wait_corrupts_c():
    """Negative control for the test above: with the A-chunk waits dropped
    (PDL_TEST_DROP_WAITS=1) the same run computes on chunks that have not landed
    and the oracle check fails -- the ordering test can see a missing wait."""
    r = _run_rc(4, "f64", 1000, 700, 300, 64,
                env_extra={"PDL_TEST_EXCHANGE_DELAY_US": "3000", "PDL_OVERLAP_A": "1", "PDL_TEST_DROP_WAITS": "1"})
    assert r.returncode != 0 or "ok=False" in r.stdout, r.stdout[-2000:]


@pytest.mark.parametrize("G,variant", [(2, None), (8, None), (4, "ozaki2"), (8, "ozaki2")])
def test_prepared_a_chunks_bitwise(G, variant, monkeypatch):
    """Variants with an A preparation exchange PREPARED A chunks (PDL_TASK_PREP_A:
    FP32 TF32 hi/lo rows; Ozaki-II residues, scales and certificate sums), so each
    Worker prepares only its own chunk: the chunk launches on the prepared panel
    (task_matmul_prepared) give bitwise the raw-panel C, serial or on side
    streams, for every Worker position -- Ozaki-II with adversarial rows whose
    elements its certificate sends to the K1 recompute over the raw rows."""
    import numpy as np

    sys.path.insert(0, ROOT)
    from paper_conf_ipps_sandrieserbp11_b200 import pdl, runtime

    M, N, K, tile = 1500, 1100, 260, 128
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    monkeypatch.setenv("PDL_DRY_RUN", "1")
    pdl.load(pdl.descriptor_path(G))
    try:
        wps = [runtime.worker_plan(M, N, K, tile, r) for r in range(G)]
    finally:
        pdl.unload()
        monkeypatch.delenv("PDL_DRY_RUN")
    torch = pytest.importorskip("torch")
    rng = np.random.default_rng(9)
    npdt, tdt = (np.float64, torch.float64) if variant else (np.float32, torch.float32)
    A = torch.from_numpy(rng.uniform(-1, 1, (M, K)).astype(npdt))
    B = torch.from_numpy(rng.uniform(-1, 1, (K, N)).astype(npdt))
    if variant:
        for i in (7, 700, 1400):
            A[i, :] = 0.0
            A[i, :2] = torch.tensor([2.0 ** 60, 1.0], dtype=tdt)
        B[:2, 11] = torch.tensor([0.0, 1.0], dtype=tdt)
    dev = torch.device("cuda", 0)
    pdl.load(pdl.descriptor_xml(1, props={"DGEMM_VARIANT": variant}) if variant else pdl.descriptor_path(1))
    try:
        pb, needs_raw = runtime.prepared_info(tdt, K, dev)
        if variant:
            assert pb > 0 and needs_raw
        else:
            assert pb == 2 * ((K + 31) // 32 * 32) * 4 and not needs_raw
            assert runtime.prepared_bytes(torch.float64, K, dev) == 0     # dmma exchanges raw rows
        for wp in wps:
            raw = runtime.PanelBuffers(wp, tdt, dev)
            prep = runtime.panel_buffers(wp, tdt, dev)
            raw.A.zero_()
            raw.A[: wp.rows].copy_(A[wp.row0: wp.row1])
            for b in (raw, prep):
                b.B[: wp.K].copy_(B[:, wp.col0: wp.col1])
            if prep.Araw is not None:
                prep.Araw.copy_(raw.A)
            pdl.set_stream(torch.cuda.current_stream())
            for j in range(wp.Gc):   # every chunk prepared (here on one Worker)
                pdl.prepare_a(raw.A[j * wp.qa:(j + 1) * wp.qa], prep.A[j * wp.qa:(j + 1) * wp.qa])
            pdl.run()
            out = []
            for bufs, conc in ((raw, False), (prep, False), (prep, True)):
                C = torch.full((wp.rows, wp.cols), float("nan"), dtype=tdt, device=dev)
                runtime.compute_groups(wp, bufs, bufs.B[: wp.K], runtime.chunk_task(C, wp, tile), {}, conc)
                pdl.sync()
                torch.cuda.synchronize()
                out.append(C.cpu())
            assert torch.equal(out[0], out[1]) and torch.equal(out[0], out[2]), (wp.r, wp.c)
    finally:
        pdl.unload()


def test_prep_a_errors():
    sys.path.insert(0, ROOT)
    torch = pytest.importorskip("torch")
    from paper_conf_ipps_sandrieserbp11_b200 import pdl
    pdl.load(pdl.descriptor_path(1))
    try:
        A = torch.rand((64, 96), dtype=torch.float64, device="cuda")
        out = torch.empty((64, 2048), dtype=torch.uint8, device="cuda")
        pdl.prepare_a(A, out)
        with pytest.raises(pdl.PDLError) as e:
            pdl.run()
        assert e.value.code == pdl.PDL_EUNSUPPORTED      # FP64 dmma exchanges raw rows
    finally:
        pdl.unload()
    pdl.load(pdl.descriptor_xml(1, props={"DGEMM_VARIANT": "ozaki2"}))
    try:
        Ap = torch.zeros((64, 4096), dtype=torch.uint8, device="cuda")
        Bd = torch.rand((96, 32), dtype=torch.float64, device="cuda")
        C = torch.empty((64, 32), dtype=torch.float64, device="cuda")
        pdl.task_matmul(Ap, Bd, C, M=64, N=32, K=96, local=True, prepared_a=True)
        with pytest.raises(pdl.PDLError) as e:
            pdl.run()
        assert e.value.code == pdl.PDL_EINVAL            # the certificate recomputes from raw rows: none given
    finally:
        pdl.unload()
