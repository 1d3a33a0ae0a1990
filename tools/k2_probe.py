"""K2 (FP32 CTA-pair kernel) timing at arbitrary shapes (development aid): device-
resident operands, CUDA-event kernel times from libpdl, the tcgen05 issue-rate floor
beside them.  python tools/k2_probe.py M N K [M N K ...]  (env PDL_SGEMM_VARIANT,
PDL_K2_DEBUG, PDL_K2_BK apply; PROBE_SMS=n runs the Worker on an n-SM partition)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402

RATE = 1111e12   # TF32(-equivalent) issue rate, profiles/r02_tc_microbench.json


def probe(M, N, K, reps=5):
    A = torch.rand(M, K, device="cuda")
    B = torch.rand(K, N, device="cuda")
    C = torch.empty(M, N, device="cuda")
    sms = int(os.environ.get("PROBE_SMS", "0"))   # > 0: one Worker on a green-context partition
    pdl.load(pdl.partition_descriptor_xml([sms]) if sms else pdl.descriptor_path(1))
    pdl.set_stream(torch.cuda.current_stream())
    for _ in range(2):
        pdl.task_matmul(A, B, C)
        pdl.run_async()
    pdl.sync()
    pdl.kernel_times()
    for _ in range(reps):
        pdl.task_matmul(A, B, C)
        pdl.run_async()
    pdl.sync()
    kt = pdl.kernel_times()
    pdl.unload()
    ms = sum(kt) / len(kt)
    mix = os.environ.get("PDL_SGEMM_VARIANT", "tf32bf16") != "3xtf32"
    floor = (2 if mix else 3) * 2.0 * M * N * K / RATE * 1e3
    return {"M": M, "N": N, "K": K, "variant": "tf32bf16" if mix else "3xtf32",
            "debug": os.environ.get("PDL_K2_DEBUG", "0"), "sms": sms or 148, "kernel_ms": round(ms, 3),
            "issue_floor_ms": round(floor, 3), "frac": round(floor / ms, 4)}


if __name__ == "__main__":
    a = [int(x) for x in sys.argv[1:]] or [16384, 16384, 16384]
    for i in range(0, len(a), 3):
        print(json.dumps(probe(*a[i:i + 3])), flush=True)
