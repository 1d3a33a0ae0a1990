"""One task through libpdl for compute-sanitizer (memcheck / racecheck /
synccheck) runs: `python tools/sanitize_run.py <variant> <M> <N> <K> [workers]`
with variant in dmma | tf32bf16 | 3xtf32 | ozaki2 | ozaki2-uniform (non-negative operands: the
certificate in the CRT pass, R23) | ozaki2-mixed (some rows / columns mix signs: both
certificates, the GEMM epilogue's per-lane column bits) | ozaki2-flagged (adversarial inputs that
send elements through the certificate's K1 recompute) | exchange (host operands,
8 Workers, the Worker<->Worker peer-copy path).  Checks the result against the
oracle on a few rows so a silent corruption under the tool also fails."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402


def main():
    variant = sys.argv[1]
    M, N, K = (int(x) for x in sys.argv[2:5])
    workers = int(sys.argv[5]) if len(sys.argv) > 5 else 1
    os.environ.pop("PDL_DRY_RUN", None)
    os.environ["PDL_ALLOW_OVERSUBSCRIBE"] = "1"
    dt = np.float32 if variant in ("3xtf32", "tf32bf16") else np.float64
    A = W.signed((M, K), dt, 1)
    B = W.signed((K, N), dt, 2)
    if variant == "ozaki2-flagged":
        A[3, :2] = [2.0 ** 60, 1.0]
        B[:2, 5] = [0.0, 1.0]
    if variant in ("ozaki2-uniform", "ozaki2-mixed"):
        A, B = np.abs(A), np.abs(B)
        A[3, :2] = [2.0 ** 60, 1.0]
        A[3, 2:] = 0.0
        B[:2, 5] = [0.0, 1.0]
        if variant == "ozaki2-mixed":
            A[10:60] *= np.where(np.random.default_rng(3).random((50, K)) < 0.5, -1.0, 1.0)
            B[:, 20:40] *= np.where(np.random.default_rng(4).random((K, 20)) < 0.5, -1.0, 1.0)
    props = ({"DGEMM_VARIANT": "ozaki2"} if variant.startswith("ozaki2") else
             {"SGEMM_VARIANT": variant} if dt == np.float32 else None)
    pdl.load(pdl.descriptor_xml(workers, props=props) if props else pdl.descriptor_path(workers))
    if variant == "exchange":
        C = np.full((M, N), np.nan, dtype=dt)
        pdl.task_matmul(A, B, C, tile=128)
        pdl.run()
    else:
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        dC = torch.full((M, N), float("nan"), dtype=dA.dtype, device="cuda")
        pdl.task_matmul(dA, dB, dC, tile=128)
        pdl.run()
        C = dC.cpu().numpy()
    stats = pdl.query("stats")
    pdl.unload()
    rows = np.array([0, 3, M // 2, M - 1])
    Cref, D = oracle.matmul(A, B, rows=rows)
    err = oracle.scaled_error(C[rows], Cref, D).max()
    tol = 1e-5 if dt == np.float32 else 1e-12
    print(f"sanitize_run {variant} {M}x{N}x{K} G={workers}: max err {err:.3e} ({'ok' if err <= tol else 'FAIL'})")
    print(stats)
    sys.exit(0 if err <= tol else 1)


if __name__ == "__main__":
    main()
