"""Results table over the BASELINE.json configs, 1 B200.

For each config / dtype / task variant: device-resident GFLOP/s (CUDA events,
warm-up, median of steps), e2e GFLOP/s through host pinned operands, max
scaled error against the oracle on sampled rows, and the oracle's own rate.
Multi-Worker configs run their Worker count oversubscribed on the one GPU (the
mapping and per-Worker launches are real; NVLink scaling is not measured).

    python tools/bench_table.py [--out profiles/r02_bench_table.md]
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402

# (config, dtype, Workers, variant): None = the dtype's default (FP64 dmma, FP32 tf32bf16)
ROWS = [("C1", "f64", 1, None), ("C1", "f32", 1, None), ("C1", "f32", 1, "3xtf32"),
        ("C2", "f64", 1, None), ("C2", "f32", 1, None), ("C2", "f32", 1, "3xtf32"), ("C2", "f64", 1, "ozaki2"),
        ("C3", "f64", 2, None), ("C3", "f64", 4, None), ("C3", "f32", 4, None), ("C3", "f32", 4, "3xtf32"),
        ("C3", "f64", 4, "ozaki2"), ("C0", "f64", 1, None), ("C0", "f64", 2, None), ("C0", "f64", 2, "ozaki2"),
        ("C4", "f64", 1, None), ("C4", "f32", 1, None), ("C4", "f32", 1, "3xtf32"), ("C4", "f64", 1, "ozaki2"),
        ("C5", "f64", 8, None), ("C5", "f32", 8, None), ("C5", "f32", 8, "3xtf32"), ("C5", "f64", 8, "ozaki2")]


def descriptor(G, dt, variant):
    if variant == "ozaki2":
        return pdl.descriptor_xml(G, props={"DGEMM_VARIANT": "ozaki2"})
    if variant in ("3xtf32", "tf32bf16"):
        return pdl.descriptor_xml(G, props={"SGEMM_VARIANT": variant})
    return pdl.descriptor_xml(G)


def timed(fn, steps, stream):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(steps):
        e0.record(stream)
        fn()
        e1.record(stream)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def run_row(cfg, dt, G, variant, steps):
    c = W.CONFIGS[cfg]
    npdt = np.float64 if dt == "f64" else np.float32
    A, B = W.config_inputs(cfg, npdt)
    flops = 2.0 * c.M * c.N * c.K
    os.environ["PDL_ALLOW_OVERSUBSCRIBE"] = "1"
    pdl.load(descriptor(G, dt, variant))
    stream = torch.cuda.current_stream()
    pdl.set_stream(stream)
    try:
        dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
        dC = torch.empty((c.M, c.N), dtype=dA.dtype, device="cuda")

        def step():
            pdl.task_matmul(dA, dB, dC, tile=c.tile)
            pdl.run_async()
        for _ in range(2):
            step()
        torch.cuda.synchronize()
        ms = timed(step, steps, stream)
        C = dC.cpu().numpy()
        hA, hB = torch.from_numpy(A).pin_memory(), torch.from_numpy(B).pin_memory()
        hC = torch.empty((c.M, c.N), dtype=dA.dtype).pin_memory()

        def estep():
            pdl.task_matmul(hA, hB, hC, tile=c.tile)
            pdl.run()
        estep()
        ems = timed(estep, max(1, steps // 2), stream)
    finally:
        pdl.unload()
    rows = np.arange(c.M) if c.M * c.N * c.K <= 2 ** 31 else W.sampled_rows(c.M, (), c.tile, n_random=24)
    t0 = time.perf_counter()
    Cref, D = oracle.matmul(A, B, rows=rows)
    ot = time.perf_counter() - t0
    err = float(oracle.scaled_error(C[rows], Cref, D).max())
    return {"config": cfg, "M": c.M, "N": c.N, "K": c.K, "tile": c.tile, "dtype": dt, "workers": G,
            "variant": variant or ("dmma" if dt == "f64" else "tf32bf16"), "ms": round(ms, 3),
            "gflops": round(flops / ms / 1e6, 1), "e2e_gflops": round(flops / ems / 1e6, 1),
            "max_scaled_err": err, "oracle_rows": int(len(rows)),
            "oracle_gflops": round(2.0 * len(rows) * c.N * c.K / ot / 1e9, 2)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "bench_table.md"))
    ap.add_argument("--steps", type=int, default=5)
    args = ap.parse_args()
    os.environ.pop("PDL_DRY_RUN", None)
    res = []
    for r in ROWS:
        d = run_row(*r, steps=args.steps)
        print(json.dumps(d), flush=True)
        res.append(d)
    lines = ["| config | M×N×K | tile | dtype | task variant | Workers (on 1 B200) | ms | GFLOP/s | e2e GFLOP/s | max scaled err | oracle GFLOP/s (rows) |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    for d in res:
        lines.append(f"| {d['config']} | {d['M']}×{d['N']}×{d['K']} | {d['tile']} | {d['dtype']} | {d['variant']} | "
                     f"{d['workers']} | {d['ms']} | {d['gflops']} | {d['e2e_gflops']} | {d['max_scaled_err']:.2e} | "
                     f"{d['oracle_gflops']} ({d['oracle_rows']}) |")
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        f.write("\n".join(lines) + "\n")
    with open(os.path.splitext(args.out)[0] + ".jsonl", "w") as f:
        for d in res:
            f.write(json.dumps(d) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
