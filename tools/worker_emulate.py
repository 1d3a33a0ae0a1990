"""Per-Worker compute time of the multi-GPU C4 step, measured on one B200.

For G = 1, 2, 4, 8 Workers, every distinct Worker position c in its grid row
(the launch grouping of runtime.compute_groups depends on c) runs exactly the
chunk launches of runtime.exchange_overlapped on its own panels -- the
rectangle, chunk sizes and launch groups of libpdl's plan for that Worker --
with the panels already resident (the NVLink exchange is modelled separately
in tools/scaling_model.py).  Serial launches on the Worker stream and
runtime.compute_groups' own choice (side streams where libpdl reports the task
variant scratch-free, else serial) are both timed with CUDA events (median of
`--reps`), and C is compared bitwise.

    python tools/worker_emulate.py [--dtype f64] [--config C4] [--reps 3]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads as W  # noqa: E402
from paper_conf_ipps_sandrieserbp11_b200 import pdl, runtime  # noqa: E402
from bench import ClockSampler  # noqa: E402


def plans(M, N, K, tile, G):
    os.environ["PDL_ALLOW_OVERSUBSCRIBE"] = "1"
    os.environ["PDL_DRY_RUN"] = "1"
    pdl.load(pdl.descriptor_path(G))
    try:
        return [runtime.worker_plan(M, N, K, tile, r) for r in range(G)]
    finally:
        pdl.unload()
        os.environ.pop("PDL_DRY_RUN", None)


def time_worker(wp, dt, tile, concurrent, reps, raw=False):
    """The Worker's step after the exchange: (prepared-A variants) the preparation
    of its own A chunk -- the other chunks arrive prepared -- then the chunk launches
    of runtime.compute_groups."""
    dev = torch.device("cuda", torch.cuda.current_device())
    g = torch.Generator(device="cuda").manual_seed(11)
    bufs = runtime.panel_buffers(wp, dt, dev, prepared=not raw)
    prep = bufs.prepared
    Araw = torch.empty((wp.Gc * wp.qa, wp.K), dtype=dt, device=dev).uniform_(generator=g)
    bufs.B.uniform_(generator=g)
    if prep:
        pdl.prepare_a(Araw, bufs.A)   # the chunks the other Workers prepared (untimed)
        pdl.run()
        if bufs.Araw is not None:     # raw rows for the certificate's recompute (landed)
            bufs.Araw.copy_(Araw)
    else:
        bufs.A.copy_(Araw)
    qa, c = wp.qa, wp.c
    Bp = bufs.B[: wp.K]
    C = torch.full((wp.rows, wp.cols), float("nan"), dtype=dt, device=dev)
    compute = runtime.chunk_task(C, wp, tile=tile)
    main = torch.cuda.current_stream()
    pdl.set_stream(main)

    def step():
        if prep:
            pdl.prepare_a(Araw[c * qa:(c + 1) * qa], bufs.A[c * qa:(c + 1) * qa])
            pdl.run_async()
        runtime.compute_groups(wp, bufs, Bp, compute, {}, concurrent)
    for _ in range(2):
        step()
    pdl.sync()
    torch.cuda.synchronize()
    if SUSTAIN_S > 0:
        return sustained_ms(step, main), C
    ms = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(main)
        step()
        e1.record(main)
        pdl.sync()
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    ms.sort()
    return ms[len(ms) // 2], C


# --sustain S: time each Worker step back to back for >= S seconds (after as long a
# warm-up), the way every GPU of a strong-scaling run repeats its step, so a short
# G = 8 step meets the same power cap as the long G = 1 step (the INT8 / TF32 paths
# run under sw_power_cap; a few isolated short steps run at boost clocks).
SUSTAIN_S = 0.0


def sustained_ms(step, stream):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    step()
    e1.record(stream)
    pdl.sync()
    torch.cuda.synchronize()
    est = max(e0.elapsed_time(e1), 1e-3)
    n = max(3, int(SUSTAIN_S * 1e3 / est))
    for _ in range(n):   # warm-up at the sustained clock
        step()
    e0.record(stream)
    for _ in range(n):
        step()
    e1.record(stream)
    pdl.sync()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n


def time_single(wp, dt, tile, reps):
    """The Worker's whole rectangle as one task (the non-overlapped exchange:
    every A chunk landed first)."""
    dev = torch.device("cuda", torch.cuda.current_device())
    bufs = runtime.PanelBuffers(wp, dt, dev)
    bufs.A.uniform_()
    bufs.B.uniform_()
    C = torch.empty((wp.rows, wp.cols), dtype=dt, device=dev)
    Ap, Bp = bufs.A[: wp.rows], bufs.B[: wp.K]
    main_s = torch.cuda.current_stream()
    pdl.set_stream(main_s)

    def once():
        pdl.task_matmul(Ap, Bp, C, M=wp.rows, N=wp.cols, K=wp.K, tile=tile, lda=Ap.stride(0), ldb=Bp.stride(0),
                        ldc=C.stride(0), local=True)
        pdl.run_async()
    for _ in range(2):
        once()
    pdl.sync()
    torch.cuda.synchronize()
    ms = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(main_s)
        once()
        e1.record(main_s)
        pdl.sync()
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    ms.sort()
    return ms[len(ms) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dtype", choices=("f64", "f32"), default="f64")
    ap.add_argument("--config", default="C4")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--gs", default="1,2,4,8")
    ap.add_argument("--variant", default=None, help="task variant (PDL_DGEMM_VARIANT / PDL_SGEMM_VARIANT)")
    ap.add_argument("--raw", action="store_true", help="exchange raw A chunks (every Worker prepares its panel)")
    ap.add_argument("--sustain", type=float, default=0.0,
                    help="seconds of back-to-back steps per timing (sustained power-capped clock)")
    args = ap.parse_args()
    global SUSTAIN_S
    SUSTAIN_S = args.sustain
    if args.variant:
        os.environ["PDL_DGEMM_VARIANT" if args.dtype == "f64" else "PDL_SGEMM_VARIANT"] = args.variant
    c = W.CONFIGS[args.config]
    dt = torch.float64 if args.dtype == "f64" else torch.float32
    out = []
    for G in [int(x) for x in args.gs.split(",")]:
        wps = plans(c.M, c.N, c.K, c.tile, G)
        pdl.load(pdl.descriptor_path(1))
        try:
            a_ex = "raw" if args.raw or not runtime.prepared_bytes(dt, c.K, "cuda") else "prepared"
            seen = set()
            rows = []
            for wp in wps:
                key = (wp.c, wp.rows, wp.cols)
                if key in seen:
                    continue
                seen.add(key)
                t_ser, C_ser = time_worker(wp, dt, c.tile, False, args.reps, args.raw)
                C_ser = C_ser.clone()
                with ClockSampler(torch.cuda.current_device()) as clk:
                    t_con, C_con = time_worker(wp, dt, c.tile, None, args.reps, args.raw)   # libpdl decides
                ck = clk.summary() or {}
                t_one = time_single(wp, dt, c.tile, args.reps)
                flops = 2.0 * wp.rows * wp.cols * wp.K
                rows.append({"c": wp.c, "rect": [wp.rows, wp.cols], "qa": wp.qa, "serial_ms": round(t_ser, 3),
                             "concurrent_ms": round(t_con, 3), "single_launch_ms": round(t_one, 3),
                             "sm_mhz": ck.get("sm_mhz"), "clock_reasons": ck.get("reasons"),
                             "bitwise": bool(torch.equal(C_ser, C_con)),
                             "concurrent_tflops": round(flops / t_con / 1e9, 1)})
                del C_ser, C_con
                torch.cuda.empty_cache()
        finally:
            pdl.unload()
        # the variant by name (the FP32 default is tf32bf16 since round 2; older files say
        # "default" for 3xtf32)
        vname = args.variant or ("dmma" if args.dtype == "f64" else "tf32bf16")
        r = {"config": args.config, "dtype": args.dtype, "variant": vname, "G": G,
             "sustain_s": args.sustain,
             "a_exchange": a_ex,
             "grid": [wps[0].Gr, wps[0].Gc],
             "max_serial_ms": max(x["serial_ms"] for x in rows),
             "max_concurrent_ms": max(x["concurrent_ms"] for x in rows),
             "max_single_launch_ms": max(x["single_launch_ms"] for x in rows),
             "sm_mhz_worst": next(x["sm_mhz"] for x in rows if x["concurrent_ms"] == max(y["concurrent_ms"] for y in rows)),
             "workers": rows}
        print(json.dumps(r), flush=True)
        out.append(r)
    t1 = out[0]["max_concurrent_ms"] if out[0]["G"] == 1 else None
    if t1:
        for r in out:
            r["compute_speedup_serial"] = round(t1 / r["max_serial_ms"], 2)
            r["compute_speedup_concurrent"] = round(t1 / r["max_concurrent_ms"], 2)
        print(json.dumps({"speedups": {r["G"]: [r["compute_speedup_serial"], r["compute_speedup_concurrent"]]
                                       for r in out}}))


if __name__ == "__main__":
    main()
