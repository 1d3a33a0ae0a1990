"""Helper for tests/test_gpu_multirank.py (run under torchrun, one rank per
Worker): the public multi-Worker API runtime.distributed_matmul on host
operands, each rank checking its C rectangle against the oracle.

    torchrun --nproc-per-node N tests/dist_check.py f64|f32 M N K tile [gloo|nccl] [variant]
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_sandrieserbp11_b200 import pdl, runtime  # noqa: E402


def main():
    dt = np.float64 if sys.argv[1] == "f64" else np.float32
    M, N, K, tile = (int(x) for x in sys.argv[2:6])
    backend = sys.argv[6] if len(sys.argv) > 6 else "gloo"
    variant = sys.argv[7] if len(sys.argv) > 7 else None
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    local = int(os.environ.get("LOCAL_RANK", "0")) % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dist.init_process_group(backend)
    os.environ.pop("PDL_DRY_RUN", None)
    pdl.load(pdl.descriptor_xml(world, variant), rank=rank, nranks=world)
    A = W.signed((M, K), dt, 501)
    B = W.signed((K, N), dt, 502)
    if os.environ.get("DIST_CHECK_ADVERSARIAL") == "1" and K >= 2:
        # elements the Ozaki-II certificate cannot certify (a 2^60 entry meeting a
        # zero of B): they go through the K1 recompute, which reads raw A rows
        for i in (3, M // 2, M - 2):
            A[i, :] = 0.0
            A[i, :2] = [2.0 ** 60, 1.0]
        B[:2, 5] = [0.0, 1.0]
    C = np.full((M, N), np.nan, dtype=dt)
    wp = runtime.distributed_matmul(torch.from_numpy(A), torch.from_numpy(B), torch.from_numpy(C), tile=tile)
    rows = np.arange(wp.row0, wp.row1)
    ok = True
    err = 0.0
    if len(rows) and wp.cols:
        Cref, D = oracle.matmul(A, B, rows=rows)
        e = oracle.scaled_error(C[wp.row0:wp.row1, wp.col0:wp.col1], Cref[:, wp.col0:wp.col1],
                                D[:, wp.col0:wp.col1])
        err = float(e.max())
        ok = err <= (1e-12 if dt == np.float64 else 1e-5)
        if not ok:
            bad = np.argwhere(~(e <= (1e-12 if dt == np.float64 else 1e-5)))
            print(f"dist_check rank {rank} rect {wp.row0}:{wp.row1} x {wp.col0}:{wp.col1}: {len(bad)} bad, "
                  f"first {bad[:5].tolist()} err {err:.3e}", file=sys.stderr, flush=True)
    t = torch.tensor([0.0 if ok else 1.0, err])
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if rank == 0:
        print(f"dist_check world={world} Gr={wp.Gr} Gc={wp.Gc} max_err={t[1].item():.3e} ok={t[0].item() == 0}")
    pdl.unload()
    dist.destroy_process_group()
    sys.exit(0 if t[0].item() == 0 else 1)


if __name__ == "__main__":
    main()
