"""CTA-shape sweep (development aid): device-resident task_matmul with the
tile kernel's shape forced each way, then the automatic choice; checks that the
shapes give bitwise the same C and prints one JSON line per problem.
FP64 K1: PDL_K1_BM = 128 / 64.  FP32 K2 (argv[2] == "f32"): PDL_K2 = 2sm / 1sm."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_sandrieserbp11_b200 import pdl

SHAPES = [(1024, 1024, 1024), (2048, 2048, 2048), (3072, 3072, 3072), (4096, 4096, 4096), (2048, 4096, 4096),
          (2048, 2048, 4096), (1250, 7000, 3000), (10000, 7000, 3000), (512, 512, 8192), (8192, 8192, 8192)]


def time_one(A, B, C, M, N, K, reps):
    s = torch.cuda.current_stream()
    pdl.set_stream(s)
    for _ in range(2):
        pdl.task_matmul(A, B, C, M, N, K, tile=0); pdl.run_async()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        pdl.task_matmul(A, B, C, M, N, K, tile=0); pdl.run_async()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    shapes = SHAPES
    if len(sys.argv) > 1 and sys.argv[1] != "default":
        shapes = [tuple(int(v) for v in s.split("x")) for s in sys.argv[1].split(",")]
    f32 = len(sys.argv) > 2 and sys.argv[2] == "f32"
    dt = torch.float32 if f32 else torch.float64
    knob, opts = ("PDL_K2", ("2sm", "1sm")) if f32 else ("PDL_K1_BM", ("128", "64"))
    pdl.load(pdl.descriptor_path(1))
    for (M, N, K) in shapes:
        g = torch.Generator(device="cuda").manual_seed(7)
        A = torch.rand(M, K, dtype=dt, device="cuda", generator=g)
        B = torch.rand(K, N, dtype=dt, device="cuda", generator=g)
        reps = max(3, int(2e11 / (2 * M * N * K)))
        out = {"M": M, "N": N, "K": K, "dtype": str(dt)}
        ref = None
        for bm in opts + ("auto",):
            if bm == "auto":
                os.environ.pop(knob, None)
            else:
                os.environ[knob] = bm
            C = torch.empty(M, N, dtype=dt, device="cuda")
            ms = time_one(A, B, C, M, N, K, reps)
            out[f"tflops_{bm}"] = round(2 * M * N * K / ms / 1e9, 1)
            if ref is None:
                ref = C.clone()
            else:
                out[f"bitwise_{bm}"] = bool(torch.equal(ref, C))
        print(json.dumps(out), flush=True)
    pdl.unload()


if __name__ == "__main__":
    main()
