"""Pinned host <-> device copy bandwidth on this box (the e2e legs' PCIe floor):
contiguous 1 GiB H2D / D2H, both directions at once, and the 2-D copy shape of the
pipelined B column panels (K rows of 16 KiB).  CUDA events; JSON line on stdout."""
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
    # B column panel of the pipelined staging: 16384 rows x 4096 fp32 out of 16384
    K, N, w = 16384, 16384, 4096
    hb = h[: K * N // 4 * 4].view(-1)[: K * (N // 4)]   # reuse the pinned buffer
    hB = h.view(-1)[: K * N // 4].view(K // 4, N)       # 4096 x 16384 view
    dB = d.view(-1)[: (K // 4) * w].view(K // 4, w)
    out["h2d_2d_panel_gbs"] = (K // 4) * w * 4 / timed(lambda: dB.copy_(hB[:, :w], non_blocking=True)) / 1e9
    del hb
    print(json.dumps({k: round(v, 2) for k, v in out.items()}))


if __name__ == "__main__":
    main()
