#!/usr/bin/env python
"""Benchmark of the PDL-mapped blocked matmul (BASELINE.json metric:
"matmul GFLOP/s at 1/2/4/8 B200 and % of tensor-core peak").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--dtype f64|f32]
                    [--config C4] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...      (one process per GPU)

A step is one pass of the whole hot path over one batch
of synthetic input: at N = 1 one FP64 DGEMM task (paper's precision,
PAPER.md L1402-1406) of config C4 (16384^3, tile 1024) through
task_matmul + pdl_run; at N > 1 the operand-panel exchange over NCCL
(all-gather in grid rows / columns) followed by each Worker's rectangle.
Strong scaling: the same 16384^3 problem is split over the N Workers.

Timed region (value): operands resident in HBM (N = 1: whole matrices; N > 1:
each Worker's unique chunks), W warm-up steps, then K steps bracketed by a
barrier + torch.cuda.synchronize(), CUDA events on the launching stream, max
over ranks.  Inputs (6 GiB FP64) are far larger than the 126 MB L2.
e2e: the same metric with host (pinned) operands through the public API,
host<->device copies inside the timed region.

Rank 0 prints ONE JSON line.  --impl reference times the CPU oracle
(oracle/, a plain triple loop accumulating in double) on a bounded row sample
of the same workload -- the reference arm of this tier.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "matmul GFLOP/s at 1/2/4/8 B200 and % of tensor-core peak"
PROFILES = os.path.join(ROOT, "profiles")
# FP64 DMMA peak measured on this box class with tools/microbench (mma.sync
# m8n8k4 from registers, 148 x 2 CTAs): profiles/r01_microbench.json.
FP64_DMMA_PEAK_TFLOPS = 37.0
# tcgen05 kind::tf32 issue rate (M=256 N=256 cta_group::2 and M=128 N=256
# cta_group::1, 148 SMs, no memory traffic): profiles/r01_tc_microbench.json.
TF32_TCGEN05_PEAK_TFLOPS = 1107.0
INT8_TCGEN05_PEAK_TOPS = 4571.0


# The paper's own result and hardware, quoted as context: it
# reports speedups only (Fig. 5), whose values PAPER.md does not retain.
PAPER_CONTEXT = {
    "workload": "FP64 DGEMM of two 8192x8192 matrices (PAPER.md L1402-1406)",
    "hardware": "2x Xeon X5550 (8 cores) + GTX 480 + GTX 285, CUBLAS DGEMM / GotoBLAS2 under StarPU "
                "(L1396-1431)",
    "published": "speedup over a single-threaded program only (Fig. 5); the values are not recoverable "
                 "from PAPER.md",
    "box_fp64_peak_gflops_derived": 340,
}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--dtype", choices=("f64", "f32"), default="f64")
    p.add_argument("--config", default="C4")
    p.add_argument("--impl", choices=("ours", "reference"), default="ours")
    p.add_argument("--e2e-steps", type=int, default=None, help="default: --steps")
    p.add_argument("--cpu-seconds", type=float, default=12.0, help="oracle sample budget")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cublas", action="store_true")
    p.add_argument("--variant", choices=("default", "ozaki2", "tf32bf16", "3xtf32"), default="default",
                   help="task variant pinned in the PDL descriptor: default (FP64 K1 DMMA / FP32 K3+K2 3xTF32) "
                        "or ozaki2 (FP64 only: K6/K7 Ozaki scheme II, INT8 residue GEMMs + CRT, with its "
                        "certificate and K1 recompute, DESIGN.md R21); FP32: tf32bf16 (the default: TF32 main "
                        "product + two BF16 correction products, DESIGN.md R22) or 3xtf32")
    p.add_argument("--no-alt", action="store_true", help="skip timing the other task variants")
    p.add_argument("--dist-backend", choices=("auto", "nccl", "gloo"), default="auto",
                   help="auto: NCCL when every rank has its own GPU, else gloo (ranks share GPUs: "
                        "validates the N>1 flow only)")
    p.add_argument("--no-f32", action="store_true", help="skip the FP32 3xTF32 leg of the FP64 N=1 line")
    return p.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except OSError:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


def tensor_peak(dtype):
    """Precision-matched tensor-core peak (TFLOP/s) and where it comes from.

    Both are MEASURED on this box class by issue-rate microbenchmarks (operands
    in registers / shared memory, no DRAM traffic): tools/microbench (DMMA) and
    tools/tc_microbench (tcgen05 kind::tf32).  The rule-of-thumb alternative
    for TF32 -- MEASURED_PEAKS bf16 burst x nominal 1.1/2.25 -- is reported
    beside it; it is lower than what tcgen05 issues, so the measured figure is
    the conservative denominator.
    """
    pk, src = peaks()
    sus = pk.get("bf16_tflops_sustained")
    if dtype == "i8":
        alt = {"peak": round(pk["bf16_tflops"] * 2, 1), "source": f"{src} bf16 burst x nominal 4.5/2.25"}
        if sus:
            alt["peak_sustained"] = round(sus * 2, 1)
        return INT8_TCGEN05_PEAK_TOPS, ("INT8 tcgen05 issue rate measured (tools/tc_microbench; "
                                        "profiles/r01_tc_microbench.json)"), alt
    if dtype == "f64":
        return FP64_DMMA_PEAK_TFLOPS, "FP64 DMMA.8x8x4 issue rate measured (tools/microbench; profiles/r01_microbench.json)", None
    alt = {"peak": round(pk["bf16_tflops"] * 1.1 / 2.25, 1),
           "source": f"{src} bf16 burst {pk['bf16_tflops']} x nominal 1.1/2.25"}
    if sus:
        alt["peak_sustained"] = round(sus * 1.1 / 2.25, 1)
    return TF32_TCGEN05_PEAK_TFLOPS, ("TF32 tcgen05 issue rate measured (tools/tc_microbench; "
                                      "profiles/r01_tc_microbench.json)"), alt


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.path = None

    def __enter__(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
            time.sleep(0.3)
        except OSError:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.2)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.path or not os.path.exists(self.path):
            return None
        rows = []
        for line in open(self.path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                try:
                    pw = float(parts[3])
                except ValueError:
                    pw = float("nan")
                rows.append((float(parts[1]), float(parts[2]), parts[5:9], pw))
            except ValueError:
                continue
        os.unlink(self.path)
        if not rows:
            return None
        maxmhz = max(r[1] for r in rows)
        loaded = [r for r in rows if r[0] > 0.5 * maxmhz] or rows
        names = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")
        reasons = sorted({names[i] for r in rows for i in range(4) if r[2][i].lower() == "active"})
        out = {"sm_mhz": float(np.median([r[0] for r in loaded])), "sm_max_mhz": maxmhz,
               "reasons": reasons, "samples": len(rows)}
        pw = [r[3] for r in loaded if r[3] == r[3]]
        if pw:   # board power under load: the INT8 / TF32 paths sit at the 1000 W cap
            out["power_w"] = round(float(np.median(pw)), 1)
        return out


def ncu_traffic(dtype, cfg):
    """DRAM bytes per launch of the dominant kernel from a committed ncu capture."""
    path = os.path.join(PROFILES, "ncu_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d.get(f"{dtype}/{cfg}")
    except (OSError, ValueError):
        return None


def variant_descriptor(pdl, world, dtype, variant):
    """PDL descriptor XML with the task variant pinned as a Worker property."""
    if variant == "default":
        return pdl.descriptor_xml(world)
    if variant in ("tf32bf16", "3xtf32"):
        return pdl.descriptor_xml(world, props={"SGEMM_VARIANT": variant})
    return pdl.descriptor_xml(world, props={"DGEMM_VARIANT": "ozaki2"})


OZ2_MODULI = (256, 255, 253, 251, 247, 241, 239, 233, 229, 227, 223, 217, 211, 199)


def ozaki2_moduli(K, bits=43):
    """Moduli count and scaling bits of ozaki2_plan (k_ozaki2.cu): the fewest
    moduli whose product M admits p >= bits with 2^(2p+1+ceil(log2 Kc)) < M."""
    nch = max(1, -(-K // 65536))
    kc = max(128, -(-(-(-K // nch)) // 128) * 128)
    lk = (kc - 1).bit_length()
    M = 1
    for n, m in enumerate(OZ2_MODULI, 1):
        M *= m
        p = max([q for q in range(1, 53) if (1 << (2 * q + 1 + lk)) < M] or [0])
        if p >= bits:
            break
    return n, p, nch, kc


# co-resident CTA pairs of the persistent K6 kernel on a B200 (148 SMs, one
# 2-CTA cluster per SM pair; grid (148, 1, 1) in profiles/r01_launches_oz2.csv)
OZ2_CLUSTERS = 74


def ozaki2_ops(rows, cols, K):
    n, p, nch, kc = ozaki2_moduli(K)
    # the n residue GEMMs and the certificate GEMM (one K chunk: K <= 65536)
    ops = 2.0 * rows * cols * kc * nch * (n + 1)
    from paper_conf_ipps_sandrieserbp11_b200 import pdl
    per_chunk = json.loads(pdl.query(f"ozaki2_launches/{rows}/{cols}/{n + 1}/{OZ2_CLUSTERS}"))
    return ops, (f"K6 oz2_gemm_persistent_kernel: {n} residue GEMMs + 1 certificate GEMM in "
                 f"{len(per_chunk) * nch} persistent launch(es) of {per_chunk} items "
                 f"(tcgen05 kind::i8, p = {p}) + CRT pass + K1 recompute of uncertified elements")


def variant_ops(variant, rows, cols, K):
    return ozaki2_ops(rows, cols, K)


def ozaki2_skip_adjust(ops, kname, guard, K):
    """The certificate GEMM is skipped when no row or column of the launch mixes signs
    (R23; stats of the last step): count n GEMMs instead of n + 1."""
    skipped = sum(w.get("certificate_gemms_skipped", 0) for w in guard)
    if skipped:
        n_mod = ozaki2_moduli(K)[0]
        ops *= n_mod / (n_mod + 1)
        kname = kname.replace("+ 1 certificate GEMM", "(the certificate GEMM skipped: no row or column mixes "
                                                      "signs, the CRT pass certifies, R23)")
    return ops, kname, skipped


def variant_label(variant, dtype, K):
    n = ozaki2_moduli(K)[0]
    return f"{dtype}-ozaki2-i8x{n}", f"ozaki2 (K6/K7, {n} moduli + certificate GEMM, CRT, K1 recompute)"


def edge_waste(rows, cols, dtype, ozaki):
    """Percent of the MMA work spent on padding of partial edge tiles (SURVEY
    8(d)): K1 computes 128 x 128 CTA tiles, K2 / K4 / K6 256 x 256 (or 256 x 512)
    CTA-pair tiles."""
    e_m, e_n = (128, 128) if dtype == "f64" and not ozaki else (256, 256)
    padded = -(-rows // e_m) * e_m * (-(-cols // e_n) * e_n)
    return round(100.0 * (padded / max(1, rows * cols) - 1.0), 3)


def host_inputs(cfg, np_dtype):
    return W.config_inputs(cfg, np_dtype)


def host_cores():
    """Host cores this process may run on.  The oracle gets them explicitly:
    torchrun sets OMP_NUM_THREADS=1 for N > 1, which would otherwise leave the
    reference arm (rank 0 alone) on one core."""
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:
        return max(1, os.cpu_count() or 1)


def cpu_baseline(A, B, seconds):
    """Time the oracle (as it stands) on a bounded row sample of the workload."""
    import oracle
    M, K = A.shape
    N = B.shape[1]
    nt = host_cores()
    rng = np.random.Generator(np.random.PCG64(99))
    ncal = 2 * nt                            # one calibration row pair per thread
    t0 = time.perf_counter()
    oracle.matmul(A, B, rows=rng.integers(0, M, size=ncal), with_mag=False, nthreads=nt)
    t1 = time.perf_counter()
    per_row = max((t1 - t0) / ncal, 1e-6)
    nrows = int(max(2, min(M, seconds / per_row)))
    rows = rng.integers(0, M, size=nrows)
    t0 = time.perf_counter()
    oracle.matmul(A, B, rows=rows, with_mag=False, nthreads=nt)
    dt = time.perf_counter() - t0
    gflops = 2.0 * nrows * N * K / dt / 1e9
    return {"value": round(gflops, 3), "unit": "GFLOP/s", "cores": nt, "kind": "oracle",
            "sample": f"{nrows} random rows x all {N} columns of the {M}x{N}x{K} product "
                      f"({2.0 * nrows * N * K:.3g} FLOP, {dt:.1f} s, double accumulation)"}


def run_reference(args):
    """Reference arm: the CPU oracle on the box's host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    c = W.CONFIGS[args.config]
    np_dtype = np.float64 if args.dtype == "f64" else np.float32
    A, B = host_inputs(args.config, np_dtype)
    import oracle
    nt = host_cores()
    rng = np.random.Generator(np.random.PCG64(5))
    per_step = max(2.0, min(20.0, 150.0 / max(1, args.steps + args.warmup)))
    ncal = 2 * nt
    t0 = time.perf_counter()
    oracle.matmul(A, B, rows=rng.integers(0, c.M, size=ncal), with_mag=False, nthreads=nt)
    per_row = max((time.perf_counter() - t0) / ncal, 1e-6)
    nrows = int(max(1, min(c.M, per_step / per_row)))
    flops = 2.0 * nrows * c.N * c.K
    for _ in range(args.warmup):
        oracle.matmul(A, B, rows=rng.integers(0, c.M, size=nrows), with_mag=False, nthreads=nt)
    times = []
    for _ in range(args.steps):
        rows = rng.integers(0, c.M, size=nrows)
        t0 = time.perf_counter()
        oracle.matmul(A, B, rows=rows, with_mag=False, nthreads=nt)
        times.append(time.perf_counter() - t0)
    ms = 1e3 * sum(times) / len(times)
    value = flops / (ms / 1e3) / 1e9
    line = {"metric": METRIC, "value": round(value, 3), "unit": "GFLOP/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": args.dtype,
            "data": "synthetic", "impl": "reference",
            "config": {"workload": f"{args.config} {c.M}x{c.N}x{c.K} ({args.dtype}), oracle row sample",
                       "M": c.M, "N": c.N, "K": c.K, "tile": c.tile, "rows_per_step": nrows},
            "cpu_baseline": {"value": round(value, 3), "unit": "GFLOP/s", "cores": nt,
                             "kind": "oracle",
                             "sample": f"{nrows} random rows x {c.N} columns per step (K={c.K})"},
            "e2e": {"value": round(value, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def spawn_ranks(args):
    """`python bench.py --gpus N` with N > 1 and no torchrun environment: start
    N ranks under torch.distributed.run (one process per GPU, rendezvous on
    127.0.0.1) with the same arguments; rank 0 prints the JSON line."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd, cwd=ROOT)


def setup_dist(args, torch, dist):
    """Rank / device / process group of this process.  --dist-backend auto:
    NCCL when every rank has its own GPU, else gloo with the ranks sharing
    devices (validates the N > 1 flow; its timings are not a scaling number)."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    ndev = torch.cuda.device_count()
    backend = args.dist_backend
    if backend == "auto":
        backend = "nccl" if ndev >= world else "gloo"
    shared = ndev < world
    if shared and backend == "nccl":
        raise SystemExit(f"{world} NCCL ranks need {world} GPUs ({ndev} visible): use --dist-backend gloo")
    local = local % ndev   # gloo validation: several ranks may share one GPU
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if backend == "nccl":
            try:
                dist.init_process_group("nccl", device_id=dev)
            except Exception as e:   # noqa: BLE001 -- reported in the line, not hidden
                # every rank sees the same failure (NCCL's init is collective): fall back to
                # gloo with host-staged exchange so the run still yields a (labelled) line
                print(f"bench.py rank {rank}: NCCL init failed ({type(e).__name__}: {e}); using gloo",
                      file=sys.stderr, flush=True)
                if dist.is_initialized():
                    dist.destroy_process_group()
                dist.init_process_group("gloo")
                backend = "gloo (NCCL init failed)"
        else:
            dist.init_process_group("gloo")
    return world, rank, local, dev, backend, shared


def device_timed(torch, dist, step, steps, stream, world, dev, local, sync):
    """K steps bracketed by barrier + synchronize on both sides, CUDA events on
    the launching stream, nvidia-smi clocks sampled during the region; returns
    (max-over-ranks ms, clocks)."""
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(steps):
            step()
        e1.record(stream)
        sync()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ms], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    return ms, clk.summary()


def k_roofline(ktimes, steps, pipe_flops, peak_dtype, kname, traffic_key, cfg, alg_bytes, rows, cols, dtype, ozaki):
    """roofline object of the dominant kernel: algorithmic work per step over
    its device time per step (CUDA events around every launch, summed over the
    Worker's chunk launches at N > 1)."""
    kavg = float(np.sum(ktimes)) / steps if ktimes else None
    peak_tf, peak_src, peak_alt = tensor_peak(peak_dtype)
    achieved = pipe_flops / (kavg / 1e3) / 1e12 if kavg else None
    r = {"bound": "tensor", "achieved": round(achieved, 2) if achieved else None,
         "peak": round(peak_tf, 1), "unit": "TFLOP/s",
         "frac": round(achieved / peak_tf, 4) if achieved else None,
         "traffic": ncu_traffic(traffic_key, cfg),
         "traffic_source": "ncu --set full capture of this kernel (profiles/ncu_traffic.json), per launch",
         "kernel": kname, "kernel_ms": round(kavg, 3) if kavg else None,
         "algorithmic_flops_per_launch": pipe_flops,
         "algorithmic_dram_bytes_per_launch": int(alg_bytes),
         "edge_waste_pct": edge_waste(rows, cols, dtype, ozaki),
         "peak_source": peak_src}
    if peak_alt:
        r["peak_alt"] = peak_alt
    return r


def clock_context(roof, clocks):
    """The peaks are issue rates at the maximum SM clock; a power-capped kernel runs
    at a lower one.  Report the fraction of the peak scaled to the median SM clock
    measured during the timed region beside the headline fraction (context only:
    `frac` stays against the fixed measured peak)."""
    if roof and roof.get("achieved") and clocks and clocks.get("sm_mhz") and clocks.get("sm_max_mhz"):
        f = clocks["sm_mhz"] / clocks["sm_max_mhz"]
        roof["frac_at_measured_clock"] = round(roof["achieved"] / (roof["peak"] * f), 4)
        roof["measured_clock_mhz"] = clocks["sm_mhz"]


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args))
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_sandrieserbp11_b200 import pdl, runtime

    world, rank, local, dev, backend, shared = setup_dist(args, torch, dist)
    os.environ.pop("PDL_DRY_RUN", None)
    if shared:
        os.environ["PDL_ALLOW_OVERSUBSCRIBE"] = "1"

    c = W.CONFIGS[args.config]
    M, N, K = c.M, c.N, c.K
    e2e_steps = args.e2e_steps or args.steps
    np_dtype = np.float64 if args.dtype == "f64" else np.float32
    tdt = torch.float64 if args.dtype == "f64" else torch.float32
    es = 8 if args.dtype == "f64" else 4
    A, B = host_inputs(args.config, np_dtype)

    if args.variant == "ozaki2" and args.dtype != "f64":
        sys.exit("--variant ozaki2 is an FP64 task variant")
    if args.variant in ("tf32bf16", "3xtf32") and args.dtype != "f32":
        sys.exit(f"--variant {args.variant} is an FP32 task variant")
    ozaki = args.variant == "ozaki2"
    # the task variant is pre-selected through the Worker's PDL properties (L1316-1326)
    desc = variant_descriptor(pdl, world, args.dtype, args.variant)
    if world == 1:
        pdl.load(desc)
    else:
        pdl.load(desc, rank=rank, nranks=world)
    stream = torch.cuda.current_stream()
    pdl.set_stream(stream)

    wp = runtime.worker_plan(M, N, K, c.tile, rank)
    flops_total = 2.0 * M * N * K
    flops_worker = 2.0 * wp.rows * wp.cols * K

    def barrier():
        if world > 1:
            dist.barrier()

    # ---- device-resident operands ----
    if world == 1:
        dA = torch.from_numpy(A).to(dev)
        dB = torch.from_numpy(B).to(dev)
        dC = torch.empty((M, N), dtype=tdt, device=dev)

        def step():
            pdl.task_matmul(dA, dB, dC, tile=c.tile)
            pdl.run_async()
    else:
        grid = runtime.Grid(wp.Gr, wp.Gc, rank, via_host=runtime.exchange_path() == "host")
        Ach, Bch = runtime.chunk_from_full(torch.from_numpy(A), torch.from_numpy(B), wp)
        Ach, Bch = Ach.to(dev), Bch.to(dev)
        bufs = runtime.panel_buffers(wp, tdt, dev)
        dC = torch.empty((wp.rows, wp.cols), dtype=tdt, device=dev)

        compute = runtime.chunk_task(dC, wp, tile=c.tile)

        def step():
            # B column-panel all-gather, then the A chunks broadcast while the
            # Worker's own chunk (and each landed chunk) computes
            runtime.exchange_overlapped(Ach, Bch, wp, grid, bufs, compute)

    for _ in range(args.warmup):
        step()
    pdl.sync()
    torch.cuda.synchronize()
    pdl.kernel_times()   # clear
    launches0 = pdl.query_json("stats")["total_launches"]
    ms_total, clocks = device_timed(torch, dist, step, args.steps, stream, world, dev, local, pdl.sync)
    ktimes = pdl.kernel_times()
    timed_launches = pdl.query_json("stats")["total_launches"] - launches0
    ms_step = ms_total / args.steps
    value = flops_total * args.steps / (ms_total / 1e3) / 1e9   # GFLOP/s, whole job

    # ---- roofline of the dominant kernel (K1, or K2 for FP32) ----
    peak_dtype = "i8" if ozaki else args.dtype
    if ozaki:
        pipe_flops, kname = variant_ops(args.variant, wp.rows, wp.cols, K)
        pipe_flops, kname, _ = ozaki2_skip_adjust(pipe_flops, kname, pdl.query_json("stats").get("ozaki_guard", []), K)
    else:
        f32name = "3xtf32" if args.variant == "3xtf32" else "tf32bf16"
        f32v = F32_VARIANTS[f32name]
        pipe_flops = flops_worker * (f32v[0] if args.dtype == "f32" else 1)
        kname = "K1 dgemm_k1_kernel (DMMA)" if args.dtype == "f64" else f32v[1]
    traffic_key = args.variant if ozaki else (
        "f32_tf32bf16" if args.dtype == "f32" and args.variant != "3xtf32" else args.dtype)
    roofline = k_roofline(ktimes, args.steps, pipe_flops, peak_dtype, kname, traffic_key, args.config,
                          (wp.rows * K + K * wp.cols + wp.rows * wp.cols) * es, wp.rows, wp.cols, args.dtype, ozaki)
    peak_tf = roofline["peak"]
    if args.dtype == "f32":
        roofline["note"] = f32v[2]
    if ozaki:
        roofline["note"] = ("achieved counts int8 tensor ops (one residue GEMM per modulus + the certificate "
                            "GEMM unless no row or column mixes signs (R23), 2 ops per MAC); useful FP64 FLOP = 2MNK")

    clock_context(roofline, clocks)

    # ---- e2e: host pinned operands through the public API, --steps steps ----
    e2e = None
    if not args.no_e2e:
        if world == 1:
            hA = torch.from_numpy(A).pin_memory()
            hB = torch.from_numpy(B).pin_memory()
            hC = torch.empty((M, N), dtype=tdt).pin_memory()

            def estep():
                pdl.task_matmul(hA, hB, hC, tile=c.tile)
                pdl.run_async()
            h2d = (M * K + K * N) * es
            d2h = M * N * es
        else:
            a0, a1 = wp.a_span
            b0, b1 = wp.b_span
            hAch, hBch = runtime.chunk_from_full(torch.from_numpy(A), torch.from_numpy(B), wp)
            hAch, hBch = hAch.pin_memory(), hBch.pin_memory()
            hCb = torch.empty((wp.rows, wp.cols), dtype=tdt).pin_memory()
            dAch = torch.empty_like(hAch, device=dev)
            dBch = torch.empty_like(hBch, device=dev)

            def estep():
                dAch.copy_(hAch, non_blocking=True)
                dBch.copy_(hBch, non_blocking=True)
                runtime.exchange_overlapped(dAch, dBch, wp, grid, bufs, compute)
                hCb.copy_(dC, non_blocking=True)
            h2d = ((a1 - a0) * K + (b1 - b0) * wp.cols) * es
            d2h = wp.rows * wp.cols * es

        def estep_synced():
            estep()
            pdl.sync()
            torch.cuda.synchronize()   # the step's result is on the host
        estep_synced()
        barrier()
        ems, _ = device_timed(torch, dist, estep_synced, e2e_steps, stream, world, dev, local, pdl.sync)
        e2e = {"value": round(flops_total * e2e_steps / (ems / 1e3) / 1e9, 1), "unit": "GFLOP/s",
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": round(ems / e2e_steps, 3), "steps": e2e_steps,
               "api": ("pdl.task_matmul + pdl.run on pinned host A, B, C (C ABI task_matmul_ex/pdl_run)"
                       if world == 1 else
                       "per rank: pinned host chunks -> runtime.exchange_overlapped -> pinned host C block")}
        if world == 1:
            del hA, hB, hC
        pdl.kernel_times()

    # ---- context: cuBLAS (torch.matmul) on the same device-resident operands ----
    cublas = None
    if world == 1 and not args.no_cublas:
        torch.backends.cuda.matmul.allow_tf32 = False
        torch.matmul(dA, dB, out=dC)
        torch.cuda.synchronize()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record()
        for _ in range(3):
            torch.matmul(dA, dB, out=dC)
        t1.record()
        torch.cuda.synchronize()
        cublas = round(flops_total * 3 / (t0.elapsed_time(t1) / 1e3) / 1e9, 1)

    # ---- the other task variants on the same resident operands (PDL-selected) ----
    alts = []
    others = ["ozaki2"] if args.dtype == "f64" and args.variant != "ozaki2" else []
    for av in (others if world == 1 and not args.no_alt else []):
        pdl.unload()
        pdl.load(variant_descriptor(pdl, 1, args.dtype, av))
        pdl.set_stream(stream)
        for _ in range(2):
            step()
        pdl.sync()
        torch.cuda.synchronize()
        pdl.kernel_times()
        ams, aclk = device_timed(torch, dist, step, args.steps, stream, world, dev, local, pdl.sync)
        akt = pdl.kernel_times()
        guard = pdl.query_json("stats").get("ozaki_guard", [])
        aops, akname = variant_ops(av, M, N, K)
        aops, akname, skipped = ozaki2_skip_adjust(aops, akname, guard, K)
        apeak, apsrc, _ = tensor_peak("i8")
        aach = aops / (float(np.mean(akt)) / 1e3) / 1e12 if akt else None
        adt, alabel = variant_label(av, args.dtype, K)
        alts.append({"variant": f"{alabel}: FP64 matmul on INT8 tcgen05",
                     "dtype": adt,
                     "value": round(flops_total * args.steps / (ams / 1e3) / 1e9, 1), "unit": "GFLOP/s",
                     "ms_per_step": round(ams / args.steps, 3),
                     "parity": "certified |C - AB| <= 5e-13 |A||B| per element (DESIGN.md R21; "
                               "tests/test_gpu_ozaki2.py, tests/test_ozaki2_certificate.py)",
                     "certificate": {"tiles_checked": sum(w["tiles_checked"] for w in guard),
                                     "elements_recomputed_by_k1": sum(w["elements_recomputed"] for w in guard),
                                     "launches_certified_in_crt_pass": sum(w.get("certified_in_crt", 0)
                                                                           for w in guard),
                                     "certificate_gemms_skipped": skipped},
                     "roofline": {"bound": "tensor", "achieved": round(aach, 1) if aach else None,
                                  "peak": apeak, "unit": "TFLOP/s",
                                  "frac": round(aach / apeak, 4) if aach else None,
                                  "traffic": ncu_traffic(av, args.config),
                                  "kernel": akname,
                                  "kernel_ms": round(float(np.mean(akt)), 3) if akt else None,
                                  "peak_source": apsrc},
                     "clocks": aclk})
        clock_context(alts[-1]["roofline"], aclk)

    # ---- FP32 (north star (2)): the tcgen05/TMEM 3xTF32 path K3+K2 on the same config ----
    f32 = f32_mix = None
    if world == 1 and args.dtype == "f64" and not args.no_f32:
        f32 = fp32_leg(args, torch, dist, pdl, stream, dev, local, c)
        f32_mix = fp32_leg(args, torch, dist, pdl, stream, dev, local, c, variant="tf32bf16")

    # ---- the oracle on the host cores, after the GPU timings (rank 0, every N) ----
    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        cpu = cpu_baseline(A, B, args.cpu_seconds)
    barrier()

    if rank == 0:
        workload = (f"{args.config} {M}x{N}x{K} blocked matmul, task tile {c.tile}, PDL b200_x{world}")
        line = {
            "metric": METRIC, "value": round(value, 1), "unit": "GFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": variant_label(args.variant, args.dtype, K)[0] if ozaki else args.dtype,
            "data": f"synthetic: numpy PCG64 U[0,1) seeds {W.seeds(c.cid)} ({args.dtype})",
            "config": {"workload": workload,
                       "M": M, "N": N, "K": K, "tile": c.tile, "parallelism": f"block2d {wp.Gr}x{wp.Gc}",
                       "task_variant": (variant_label(args.variant, args.dtype, K)[1] if ozaki else
                                        ("dmma (K1)" if args.dtype == "f64" else
                                         ("3xtf32" if args.variant == "3xtf32" else "tf32bf16") + " (K3+K2)")),
                       "l2": "inputs larger than L2 (operands >> 126 MB), no flush needed"},
            "pct_of_tensor_peak": round(100 * (pipe_flops / flops_worker) * value / world / (peak_tf * 1e3), 2),
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": int(timed_launches),
            "clocks": clocks,
            "paper_context": PAPER_CONTEXT,
        }
        if world > 1:
            line["config"]["dist_backend"] = backend
            if shared:
                line["config"]["note"] = (f"{world} ranks share {torch.cuda.device_count()} GPU(s) over gloo: "
                                          "validates the N>1 flow, not a scaling measurement")
        if cublas is not None:
            line["cublas_gflops_same_operands"] = cublas
        if alts:
            line["alt_variants"] = alts
        if f32 is not None:
            line["f32_3xtf32"] = f32
        if f32_mix is not None:
            line["f32_tf32bf16"] = f32_mix
        print(json.dumps(line), flush=True)
    pdl.unload()
    if world > 1:
        dist.destroy_process_group()


F32_VARIANTS = {
    # SGEMM_VARIANT -> (tensor passes per K block in TF32-equivalents, kernel label, note)
    "3xtf32": (3, "K2 gemm_3xtf32_2sm_kernel<false> (tcgen05 cta_group::2 kind::tf32 x3)",
               "achieved counts the 3 TF32 tensor products; useful FLOP = 1/3"),
    "tf32bf16": (2, "K2 gemm_3xtf32_2sm_kernel<true> (tcgen05 cta_group::2 kind::tf32 + 2x kind::f16)",
                 "achieved counts TF32-equivalent tensor work: a_hi*b_hi (TF32) + two BF16 correction "
                 "products at twice the TF32 rate = 2 TF32 passes; useful FLOP = 1/2 (DESIGN.md R22)"),
}


def fp32_leg(args, torch, dist, pdl, stream, dev, local, c, variant="3xtf32"):
    """FP32 inputs through an SGEMM task variant (K3 split + K2 tcgen05 CTA-pair
    kernel; `variant` pinned through the Worker's SGEMM_VARIANT PDL property),
    device-resident and end to end, on the same config: the tcgen05/TMEM kernel
    of north star (2) with a driver-run number."""
    M, N, K = c.M, c.N, c.K
    A, B = host_inputs(args.config, np.float32)
    passes, kname, note = F32_VARIANTS[variant]
    pdl.unload()
    pdl.load(pdl.descriptor_xml(1, props={"SGEMM_VARIANT": variant}))
    pdl.set_stream(stream)
    dA = torch.from_numpy(A).to(dev)
    dB = torch.from_numpy(B).to(dev)
    dC = torch.empty((M, N), dtype=torch.float32, device=dev)

    def step():
        pdl.task_matmul(dA, dB, dC, tile=c.tile)
        pdl.run_async()
    for _ in range(max(2, args.warmup)):
        step()
    pdl.sync()
    torch.cuda.synchronize()
    pdl.kernel_times()
    ms, clk = device_timed(torch, dist, step, args.steps, stream, 1, dev, local, pdl.sync)
    kt = pdl.kernel_times()
    flops = 2.0 * M * N * K
    roof = k_roofline(kt, args.steps, passes * flops, "f32", kname,
                      "f32" if variant == "3xtf32" else "f32_" + variant, args.config,
                      (M * K + K * N + M * N) * 4, M, N, "f32", False)
    roof["note"] = note
    out = {"value": round(flops * args.steps / (ms / 1e3) / 1e9, 1), "unit": "GFLOP/s", "dtype": "f32",
           "ms_per_step": round(ms / args.steps, 3), "task_variant": f"{variant} (K3+K2)",
           "parity": ("max rel err <= 1e-5 vs oracle (tests/test_gpu_parity.py)" if variant == "3xtf32" else
                      "max rel err <= 1e-5 vs oracle (tests/test_gpu_tf32bf16.py; split bound R22)"),
           "data": f"synthetic: numpy PCG64 U[0,1) seeds {W.seeds(c.cid)} (f32)",
           "roofline": roof, "clocks": clk}
    clock_context(roof, clk)
    if not args.no_e2e:
        hA = torch.from_numpy(A).pin_memory()
        hB = torch.from_numpy(B).pin_memory()
        hC = torch.empty((M, N), dtype=torch.float32).pin_memory()

        def estep():
            pdl.task_matmul(hA, hB, hC, tile=c.tile)
            pdl.run()
            torch.cuda.synchronize()
        estep()
        ems, _ = device_timed(torch, dist, estep, args.steps, stream, 1, dev, local, pdl.sync)
        out["e2e"] = {"value": round(flops * args.steps / (ems / 1e3) / 1e9, 1), "unit": "GFLOP/s",
                      "h2d_bytes_per_step": (M * K + K * N) * 4, "d2h_bytes_per_step": M * N * 4,
                      "ms_per_step": round(ems / args.steps, 3)}
    del dA, dB, dC
    return out


if __name__ == "__main__":
    main()
