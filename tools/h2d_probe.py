"""Pinned host <-> device copy bandwidth on this box (the e2e legs' PCIe floor):
contiguous 1 GiB H2D / D2H and both directions at once.  CUDA events; JSON line on
stdout."""
import json

import torch


def timed(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps / 1e3


def main():
    n = 1 << 28   # 1 GiB of fp32
    h = torch.empty(n, dtype=torch.float32).pin_memory()
    h2 = torch.empty(n, dtype=torch.float32).pin_memory()
    d = torch.empty(n, dtype=torch.float32, device="cuda")
    d2 = torch.empty(n, dtype=torch.float32, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    out = {}
    out["h2d_gbs"] = n * 4 / timed(lambda: d.copy_(h, non_blocking=True)) / 1e9
    out["d2h_gbs"] = n * 4 / timed(lambda: h.copy_(d, non_blocking=True)) / 1e9

    def both():
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        torch.cuda.current_stream().wait_stream(s1)
        torch.cuda.current_stream().wait_stream(s2)
    t = timed(both)
    out["duplex_total_gbs"] = 2 * n * 4 / t / 1e9
    print(json.dumps({k: round(v, 2) for k, v in out.items()}))


if __name__ == "__main__":
    main()
