"""Heterogeneous-Worker scheduling on one B200.

Two Workers on disjoint SM partitions of device 0 (green contexts from the PDL
property SM_LIMIT; default 96 + 48 SMs, the paper's fast + slow GPU pair of
L1398-1402 in miniature) run one FP64 task C = A B (device-resident operands)
under three mappings:

  block     -- equal BLOCK split (no speed knowledge): the slow Worker decides
  weighted  -- BLOCK weighted by PDL RELATIVE_SPEED (= SM ratio)
  dynamic   -- DYNAMIC: the kernels claim tiles from a shared counter

plus the whole-device one-Worker run as the reference.  Makespan = host time
of pdl_run() (launch + device sync), median of --reps after a warm-up.

    python tools/hetero_bench.py [--n 8192] [--sm 96 48] [--dtype f64|f32]
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402


def timed(desc, A, B, C, dist, reps, tile):
    pdl.load(desc)
    try:
        ts = []
        for i in range(reps + 1):
            pdl.task_matmul(A, B, C, tile=tile, dist=dist)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            pdl.run()
            t1 = time.perf_counter()
            if i:
                ts.append((t1 - t0) * 1e3)
        st = pdl.query_json("stats")
        return statistics.median(ts), st
    finally:
        pdl.unload()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=8192)
    ap.add_argument("--sm", type=int, nargs="+", default=[96, 48])
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--tile", type=int, default=256)
    ap.add_argument("--mixed", type=float, default=0.0,
                    help="also run per-Worker variants: ozaki2 on the first partition, dmma on the "
                         "others, BLOCK weighted by this RELATIVE_SPEED of the first Worker (FP64)")
    args = ap.parse_args()
    dt = torch.float64 if args.dtype == "f64" else torch.float32
    n = args.n
    g = torch.Generator(device="cuda").manual_seed(1)
    A = torch.rand((n, n), dtype=dt, device="cuda", generator=g)
    B = torch.rand((n, n), dtype=dt, device="cuda", generator=g)
    C = torch.empty((n, n), dtype=dt, device="cuda")
    ref = torch.empty_like(C)
    flops = 2.0 * n ** 3
    rows = []
    t, st = timed(pdl.descriptor_path(1), A, B, ref, None, args.reps, args.tile)
    rows.append({"mapping": "whole device, 1 Worker", "ms": t, "tflops": flops / t / 1e9})
    speeds = [s / min(args.sm) for s in args.sm]
    for name, desc, dist in (
            ("block (equal split)", pdl.partition_descriptor_xml(args.sm), None),
            ("block weighted by RELATIVE_SPEED", pdl.partition_descriptor_xml(args.sm, speeds=speeds), None),
            ("dynamic (tile claims)", pdl.partition_descriptor_xml(args.sm), "DYNAMIC")):
        t, st = timed(desc, A, B, C, dist, args.reps, args.tile)
        assert torch.equal(C, ref), f"{name}: result differs from the one-Worker run"
        r = {"mapping": name, "ms": t, "tflops": flops / t / 1e9,
             "worker_kernel_ms": [round(w["kernel_ms"], 2) for w in st["workers"]],
             "sm": [w["sm_limit"] for w in st["workers"]]}
        if "dynamic" in st:
            r["tiles"] = st["dynamic"]["tiles"]
        rows.append(r)
    if args.mixed > 0 and args.dtype == "f64":
        # the paper's premise: one task, a variant per PU pre-selected from the PDL
        oz = pdl.descriptor_xml(1, props={"DGEMM_VARIANT": "ozaki2"})
        t, st = timed(oz, A, B, C, None, args.reps, args.tile)
        rows.append({"mapping": "whole device, 1 Worker, ozaki2", "ms": t, "tflops": flops / t / 1e9})
        wp = [{"DGEMM_VARIANT": "ozaki2"}] + [{"DGEMM_VARIANT": "dmma"}] * (len(args.sm) - 1)
        sp = [args.mixed] + [s / min(args.sm[1:]) for s in args.sm[1:]]
        desc = pdl.partition_descriptor_xml(args.sm, speeds=sp, worker_props=wp)
        t, st = timed(desc, A, B, C, None, args.reps, args.tile)
        err = float(((C - ref).abs() / (A.abs() @ B.abs())).max())
        rows.append({"mapping": f"per-Worker variants (ozaki2 | dmma), weighted {sp}", "ms": t,
                     "tflops": flops / t / 1e9, "max_scaled_diff_vs_dmma": err,
                     "worker_kernel_ms": [round(w["kernel_ms"], 2) for w in st["workers"]],
                     "sm": [w["sm_limit"] for w in st["workers"]]})
    out = {"n": n, "dtype": args.dtype, "partitions": args.sm, "rows": rows}
    print(json.dumps(out))
    print(f"\n| mapping ({args.dtype} {n}^3, SMs {args.sm}) | ms | TFLOP/s | per-Worker kernel ms | tiles |")
    print("|---|---|---|---|---|")
    for r in rows:
        print(f"| {r['mapping']} | {r['ms']:.1f} | {r['tflops']:.1f} | {r.get('worker_kernel_ms', '')} | "
              f"{r.get('tiles', '')} |")


if __name__ == "__main__":
    main()
