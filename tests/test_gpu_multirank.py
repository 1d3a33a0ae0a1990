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


def _run(world, *args):
    torch = pytest.importorskip("torch")
    backend = "nccl" if torch.cuda.device_count() >= world else "gloo"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={_port()}", os.path.join(ROOT, "tests", "dist_check.py"),
           *[str(a) for a in args[:5]], backend, *[str(a) for a in args[5:]]]
    env = dict(os.environ, PDL_ALLOW_OVERSUBSCRIBE="1")
    env.pop("PDL_DRY_RUN", None)
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert "ok=True" in r.stdout


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_distributed_matmul(world, dt):
    _run(world, dt, 1000, 700, 300, 128)


def test_distributed_ragged_8():
    _run(8, "f64", 1000, 700, 300, 64)


def test_distributed_ozaki_4():
    _run(4, "f64", 777, 513, 1000, 128, "ozaki")


def test_distributed_ozaki2_4():
    _run(4, "f64", 777, 513, 1000, 128, "ozaki2")
