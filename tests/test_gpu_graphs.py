"""CUDA-graph replay of repeated tasks (PDL_TASK_GRAPH): the first run of a task
signature runs normally, the second is captured into a CUDA graph, later runs
replay it.  Replays must be bitwise equal to plain runs (the graph holds the
same launches), count the same launches, and feed pdl_kernel_times."""
import time

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402


@pytest.fixture(autouse=True)
def _env(monkeypatch):
    for k in ("PDL_DRY_RUN", "PDL_GRAPH", "PDL_PIPELINE"):
        monkeypatch.delenv(k, raising=False)
    monkeypatch.setenv("PDL_ALLOW_OVERSUBSCRIBE", "1")
    pdl.unload()
    yield
    pdl.unload()


def runs(desc, A, B, n, graph, tile=0, host=False, pinned=False):
    """n runs of one task signature; returns C after each run and the stats."""
    pdl.load(desc)
    try:
        M, N = A.shape[0], B.shape[1]
        if host:
            hA, hB = torch.from_numpy(A), torch.from_numpy(B)
            hC = torch.empty((M, N), dtype=hA.dtype)
            if pinned:
                hA, hB, hC = hA.pin_memory(), hB.pin_memory(), hC.pin_memory()
            dA, dB, dC = hA, hB, hC
        else:
            dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
            dC = torch.empty((M, N), dtype=dA.dtype, device="cuda")
        outs, launches = [], []
        for _ in range(n):
            dC.fill_(float("nan"))
            torch.cuda.synchronize()
            pdl.task_matmul(dA, dB, dC, tile=tile, graph=graph)
            pdl.run()
            outs.append(dC.cpu().numpy().copy())
            launches.append(pdl.query_json("stats")["launches"])
        kt = pdl.kernel_times()
        return outs, launches, pdl.query_json("stats")["workers"][0], kt
    finally:
        pdl.unload()


@pytest.mark.parametrize("dt,variant", [(np.float64, None), (np.float32, None), (np.float64, "ozaki2")])
def test_graph_replay_bitwise(dt, variant):
    A = W.uniform((1000, 700), dt, 1)
    B = W.uniform((700, 900), dt, 2)
    props = {}
    if variant:
        props["DGEMM_VARIANT" if dt == np.float64 else "SGEMM_VARIANT"] = variant
    desc = pdl.descriptor_xml(1, props=props)
    ref, ref_l, _, _ = runs(desc, A, B, 1, graph=False, tile=128)
    outs, launches, st, kt = runs(desc, A, B, 4, graph=True, tile=128)
    for C in outs:
        assert np.array_equal(C, ref[0])
    assert launches == [ref_l[0]] * 4
    assert st["graphs"] == 1 and st["graph_replays"] == 3
    assert len(kt) >= 4 and all(t > 0 for t in kt)
    Cref, D = oracle.matmul(A, B)
    assert oracle.scaled_error(outs[-1], Cref, D).max() <= (1e-12 if dt == np.float64 else 1e-5)


def test_graph_multiworker_pinned_pipelined(monkeypatch):
    """4 Workers, pinned host operands through the pipelined staging path
    (copy-in / copy-out / second compute stream, all joined by events).  The
    Worker<->Worker exchange (which runs uncaptured, its chunk tasks on device
    panels) is off, so each Worker stages its panels through this path."""
    monkeypatch.setenv("PDL_PIPELINE", "force")
    monkeypatch.setenv("PDL_EXCHANGE", "0")
    A = W.signed((777, 513), np.float64, 3)
    B = W.signed((513, 640), np.float64, 4)
    ref, _, _, _ = runs(pdl.descriptor_xml(4), A, B, 1, graph=False, tile=64, host=True, pinned=True)
    outs, _, st, _ = runs(pdl.descriptor_xml(4), A, B, 3, graph=True, tile=64, host=True, pinned=True)
    for C in outs:
        assert np.array_equal(C, ref[0])
    assert st["graphs"] == 1 and st["graph_replays"] == 2


def test_pageable_host_memory():
    """Pageable host operands: captured (memcpy nodes) or, where the capture
    refuses them, run uncaptured -- either way every run is correct."""
    A = W.uniform((300, 200), np.float64, 5)
    B = W.uniform((200, 260), np.float64, 6)
    outs, _, st, _ = runs(pdl.descriptor_xml(1), A, B, 3, graph=True, host=True, pinned=False)
    Cref, D = oracle.matmul(A, B)
    for C in outs:
        assert oracle.scaled_error(C, Cref, D).max() <= 1e-12
    assert st["graphs"] <= 1


def test_graph_env_and_launch_overhead(monkeypatch, capsys):
    """PDL_GRAPH=1 graphs every task; report the per-run host time of a
    launch-bound task (Ozaki II at 256^3: 17 launches) with and without."""
    A = W.uniform((256, 256), np.float64, 7)
    B = W.uniform((256, 256), np.float64, 8)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    dC = torch.empty((256, 256), dtype=torch.float64, device="cuda")
    res = {}
    for mode in ("plain", "graph"):
        if mode == "graph":
            monkeypatch.setenv("PDL_GRAPH", "1")
        pdl.load(pdl.descriptor_xml(1, props={"DGEMM_VARIANT": "ozaki2"}))
        for _ in range(3):
            pdl.task_matmul(dA, dB, dC)
            pdl.run()
        t0 = time.perf_counter()
        for _ in range(50):
            pdl.task_matmul(dA, dB, dC)
            pdl.run()
        res[mode] = (time.perf_counter() - t0) / 50 * 1e6
        st = pdl.query_json("stats")["workers"][0]
        pdl.unload()
        if mode == "graph":
            assert st["graph_replays"] >= 50
        Cref, D = oracle.matmul(A, B)
        assert oracle.scaled_error(dC.cpu().numpy(), Cref, D).max() <= 1e-12
    with capsys.disabled():
        print(f"\n[graphs] ozaki2 256^3 per-run host time: plain {res['plain']:.1f} us, graph {res['graph']:.1f} us")
