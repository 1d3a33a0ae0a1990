"""Quick device-resident timing of the libpdl tile kernels (development aid)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_sandrieserbp11_b200 import pdl

def bench(n, dt, reps=3, cublas=False):
    torch.manual_seed(0)
    A = torch.rand(n, n, dtype=dt, device="cuda"); B = torch.rand(n, n, dtype=dt, device="cuda")
    C = torch.empty(n, n, dtype=dt, device="cuda")
    s = torch.cuda.current_stream()
    pdl.load(pdl.descriptor_path(1)); pdl.set_stream(s)
    for _ in range(2):
        pdl.task_matmul(A, B, C, tile=0); pdl.run_async()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        pdl.task_matmul(A, B, C, tile=0); pdl.run_async()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    st = pdl.query_json("stats")
    pdl.unload()
    r = {"n": n, "dtype": str(dt), "ms": ms, "tflops": 2 * n**3 / ms / 1e9, "kernel_ms": st["workers"][0]["kernel_ms"]}
    if cublas:
        torch.backends.cuda.matmul.allow_tf32 = False
        for _ in range(2): torch.matmul(A, B, out=C)
        torch.cuda.synchronize(); e0.record()
        for _ in range(reps): torch.matmul(A, B, out=C)
        e1.record(); torch.cuda.synchronize()
        r["cublas_tflops"] = 2 * n**3 / (e0.elapsed_time(e1) / reps) / 1e9
    print(json.dumps(r), flush=True)

for n in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "4096,8192").split(",")]:
    bench(n, torch.float64, cublas=True)
    bench(n, torch.float32, cublas=True)
