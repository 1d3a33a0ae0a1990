"""Ozaki variant accuracy sweep (slices x rounding) against the oracle on
C4-shaped rows (K = 16384): max / mean scaled error, U[0,1) and U[-1,1)."""
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
out = []
for dist in ("uniform", "signed"):
    gen = W.uniform if dist == "uniform" else W.signed
    A = gen((M, K), np.float64, 61)
    B = gen((K, N), np.float64, 62)
    Cref, D = oracle.matmul(A, B)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    for rnd in ("trunc", "nearest"):
        for S in (5, 6, 7):
            os.environ["PDL_OZAKI_ROUNDING"] = rnd
            pdl.load(pdl.descriptor_xml(1, "ozaki", S))
            dC = torch.empty((M, N), dtype=torch.float64, device="cuda")
            pdl.task_matmul(dA, dB, dC)
            pdl.run()
            pdl.unload()
            C = dC.cpu().numpy()
            err = oracle.scaled_error(C, Cref, D)
            sg = ((C - Cref) / D).mean()
            r = {"dist": dist, "rounding": rnd, "S": S, "max_err": float(err.max()),
                 "mean_err": float(err.mean()), "mean_signed": float(sg)}
            print(json.dumps(r), flush=True)
            out.append(r)
