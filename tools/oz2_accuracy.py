"""Ozaki-II (DGEMM_VARIANT = ozaki2) accuracy sweep against the oracle on
C4-shaped rows (K = 16384): max / mean scaled error per moduli count (and the
scaling bits p the plan derives), for U[0,1), U[-1,1) and rows / columns
spread over 2^+-30.  Output: one JSON line per setting (profiles/r01_ozaki2_accuracy.txt).

    python tools/oz2_accuracy.py
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402

M, N, K = 512, 2048, 16384
for dist in ("uniform", "signed", "spread"):
    if dist == "uniform":
        A, B = W.uniform((M, K), np.float64, 61), W.uniform((K, N), np.float64, 62)
    else:
        A, B = W.signed((M, K), np.float64, 63), W.signed((K, N), np.float64, 64)
        if dist == "spread":   # per-row / per-column scales over 2^-30 .. 2^30
            A = A * np.exp2(np.linspace(-30, 30, M)).round()[:, None]
            B = B * np.exp2(np.linspace(30, -30, N)).round()[None, :]
    Cref, D = oracle.matmul(A, B)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    for nmod in (11, 12, 13, 14, 0):
        plan = json.loads(pdl.query(f"ozaki2_plan/{K}/43/{nmod}"))
        pdl.load(pdl.descriptor_xml(1, props={"DGEMM_VARIANT": "ozaki2", "OZAKI2_MODULI": nmod}))
        dC = torch.empty((M, N), dtype=torch.float64, device="cuda")
        pdl.task_matmul(dA, dB, dC)
        pdl.run()
        pdl.unload()
        C = dC.cpu().numpy()
        err = oracle.scaled_error(C, Cref, D)
        print(json.dumps({"dist": dist, "moduli": plan["n"], "auto": nmod == 0, "p": plan["p"],
                          "max_err": float(err.max()), "mean_err": float(err.mean()),
                          "mean_signed": float(((C - Cref) / np.where(D > 0, D, 1)).mean())}), flush=True)
