"""N>1 path on CPU: world_size 2 and 4 processes over gloo.

Each rank binds its Worker with pdl_load_rank (dry run: no device), takes its
BLOCK plan from libpdl, slices its unique operand chunks, and runs the real
exchange code (runtime.exchange: all-gather in grid rows / columns).  The
gathered panels must equal the A row-panel and B column-panel of the Worker's
C rectangle, and the rectangles of all ranks must tile C exactly once.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, shapes, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), PDL_DRY_RUN="1")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_sandrieserbp11_b200 import pdl, runtime
    import workloads as W
    out = []
    try:
        pdl.load(pdl.descriptor_path(world), rank=rank, nranks=world)
        assert pdl.query("local_workers") == "1"
        for (M, N, K, tile) in shapes:
            A = torch.from_numpy(W.signed((M, K), np.float64, 1))
            B = torch.from_numpy(W.signed((K, N), np.float64, 2))
            wp = runtime.worker_plan(M, N, K, tile, rank)
            grid = runtime.Grid(wp.Gr, wp.Gc, rank)
            Ach, Bch = runtime.chunk_from_full(A, B, wp)
            bufs = runtime.PanelBuffers(wp, A.dtype, A.device)
            Ap, Bp = runtime.exchange(Ach, Bch, wp, grid, bufs)
            ok_a = torch.equal(Ap, A[wp.row0:wp.row1])
            ok_b = torch.equal(Bp, B[:, wp.col0:wp.col1])
            # overlapped exchange: every chunk handed to compute() must already
            # hold its rows; own chunk first; rows covered exactly once
            bufs2 = runtime.PanelBuffers(wp, A.dtype, A.device)
            seen = []

            def compute(j, lo, hi, Arows, Bp2, first):
                seen.append((j, lo, hi, first))
                assert torch.equal(Arows, A[wp.row0 + lo: wp.row0 + hi])
                assert torch.equal(Bp2, B[:, wp.col0:wp.col1])

            Ap2, Bp2 = runtime.exchange_overlapped(Ach, Bch, wp, grid, bufs2, compute)
            ok_a = ok_a and torch.equal(Ap2, A[wp.row0:wp.row1]) and torch.equal(Bp2, Bp)
            lo_c, hi_c = runtime.chunk_rows(wp, wp.c)
            if seen:
                ok_a = ok_a and seen[0][3] and not any(s[3] for s in seen[1:])
                ok_a = ok_a and (hi_c == lo_c or seen[0][0] == wp.c)
            ok_a = ok_a and sum(s[2] - s[1] for s in seen) == (wp.rows if wp.cols else 0)
            # single launch after the whole A exchange (overlap_a=False): one call, all rows
            bufs3 = runtime.PanelBuffers(wp, A.dtype, A.device)
            seen.clear()
            runtime.exchange_overlapped(Ach, Bch, wp, grid, bufs3, compute, overlap_a=False)
            ok_a = ok_a and (seen == ([(wp.c, 0, wp.rows, True)] if wp.rows and wp.cols else []))
            out.append((M, N, K, tile, wp.row0, wp.row1, wp.col0, wp.col1, wp.Gr, wp.Gc, ok_a, ok_b))
        pdl.unload()
        q.put((rank, out, None))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, out, repr(e)))
    finally:
        dist.destroy_process_group()


SHAPES = [(64, 64, 64, 32), (100, 70, 30, 16), (37, 53, 19, 0), (129, 257, 65, 64), (3, 200, 7, 8)]


@pytest.mark.parametrize("world", [2, 4])
def test_exchange_assembles_panels(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, SHAPES, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, out, err in res:
        assert err is None, f"rank {rank}: {err}"
        assert len(out) == len(SHAPES)
    for si, (M, N, K, tile) in enumerate(SHAPES):
        cover = np.zeros((M, N), dtype=int)
        for rank, out, _ in res:
            _, _, _, _, r0, r1, c0, c1, Gr, Gc, ok_a, ok_b = out[si]
            assert ok_a and ok_b, (rank, SHAPES[si])
            assert Gr * Gc == world
            cover[r0:r1, c0:c1] += 1
        assert np.all(cover == 1)


def test_reference_arm_uses_all_host_cores():
    """bench.py --impl reference (the oracle on the host cores) under torchrun
    with 2 ranks: rank 0 alone prints one line, on every core this process may
    use, although torchrun sets OMP_NUM_THREADS=1 for N > 1."""
    import json
    import subprocess
    import sys
    env = dict(os.environ, OMP_NUM_THREADS="1")
    out = subprocess.run(
        [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
         "--master-addr", "127.0.0.1", "--master-port", "29587", os.path.join(ROOT, "bench.py"), "--gpus", "2",
         "--impl", "reference", "--config", "C1", "--steps", "1", "--warmup", "1"],
        capture_output=True, text=True, timeout=300, env=env, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2
    assert d["cpu_baseline"]["cores"] == len(os.sched_getaffinity(0))


def _stalled_peer(rank, world, port, q):
    """Rank 0 waits for a broadcast rank 1 never sends (rank 1 is stuck in host
    work): the handle's wait times out after PDL_EXCHANGE_TIMEOUT_S and the
    runtime reports it as PDL_ENCCL, the library's exchange-failure code."""
    import sys
    import time
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), PDL_EXCHANGE_TIMEOUT_S="2")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_sandrieserbp11_b200 import pdl, runtime
    res = None
    try:
        if rank == 0:
            t = torch.zeros(16)
            try:
                runtime._broadcast(t, 1, None).wait()
                res = "no error"
            except pdl.PDLError as e:
                res = e.code
        else:
            time.sleep(8)
            res = "peer"
    except Exception as e:  # pragma: no cover
        res = repr(e)
    q.put((rank, res))


def test_exchange_timeout_maps_to_pdl_enccl():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_stalled_peer, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=30)
        if p.is_alive():
            p.kill()
    from paper_conf_ipps_sandrieserbp11_b200 import pdl
    assert res[0] == pdl.PDL_ENCCL, res
