"""Strong-scaling model of the multi-Worker path (NVLink scaling is not
measurable with one GPU per gpurun call; this predicts it from measured parts).

Per Worker (plan from libpdl, dry run): compute time = the measured time of the
Worker's own chunk launches on one B200 where tools/worker_emulate.py has it
(profiles/r01_worker_emulate_*.jsonl: the worst Worker position, launch grouping
and wave quantisation included), else its FLOPs / the measured single-B200 rate
of the task variant (profiles/r01_bench_table.jsonl, C4);
exchange = B column-panel all-gather (exposed) + A-chunk broadcasts overlapped
with the chunk kernels (exposed only if a chunk transfer outlasts the previous
chunk's compute).  NVLink: 770 GB/s per direction per GPU (the measured peer
copy bandwidth quoted in /opt/skills/guides/B200_PROFILING.md), all-gather
received bytes at that rate.

    python tools/scaling_model.py   -> markdown table on stdout
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["PDL_DRY_RUN"] = "1"
from paper_conf_ipps_sandrieserbp11_b200 import pdl  # noqa: E402

NVLINK = 770e9
# the task variants of this build (Ozaki scheme I is retired)
CURRENT = {("f64", "dmma"), ("f32", "3xtf32"), ("f32", "tf32bf16"), ("f64", "ozaki2")}
CLOCK = {}   # (dtype, variant, G) -> median SM MHz during the worst Worker's timing (if recorded)


def rates():
    r = {}
    with open(os.path.join(ROOT, "profiles", "r01_bench_table.jsonl")) as f:
        for line in f:
            d = json.loads(line)
            if d["config"] == "C4" and (d["dtype"], d["variant"]) in CURRENT:
                r[(d["dtype"], d["variant"])] = d["gflops"] * 1e9
    return r


def emulated():
    """(dtype, variant, G) -> measured worst-Worker compute seconds (round-2
    measurements, which include the prepared-A exchange and the Ozaki-II
    certificate, override round 1's)."""
    out = {}
    for fn in sorted(os.listdir(os.path.join(ROOT, "profiles")), key=lambda f: (not f.startswith("r01"), f)):
        if (fn.startswith("r01_worker_emulate_") or fn.startswith("r02_worker_emulate_")) and fn.endswith(".jsonl") \
                and "_raw" not in fn:   # r02 "_raw": the raw-exchange comparison runs
            with open(os.path.join(ROOT, "profiles", fn)) as f:
                for line in f:
                    d = json.loads(line)
                    if "G" in d and d.get("config") == "C4":
                        # "default" = the FP32 default when the file was written (3xtf32 before
                        # round 2's tf32bf16; newer files name the variant)
                        var = {"default": "dmma" if d["dtype"] == "f64" else "3xtf32"}.get(
                            d.get("variant", "default"), d.get("variant"))
                        out[(d["dtype"], var, d["G"])] = d["max_concurrent_ms"] / 1e3
                        CLOCK[(d["dtype"], var, d["G"])] = d.get("sm_mhz_worst")
    return out


def a_bytes_per_elem(dt, var, K):
    """Latency-critical bytes per A element on NVLink: the prepared rows of the
    variants that exchange them (runtime.panel_buffers; pdl prepared_a): FP32
    3xTF32 TF32 hi/lo (2 Kp floats per row); FP64 Ozaki-II residues of 13 moduli +
    the certificate plane + 16 bytes of row scale / certificate sum.  Ozaki-II's
    raw rows travel after them and are read only by each chunk task's final K1
    recompute (hidden behind the residue GEMMs; not counted here).  K1: raw rows."""
    if dt == "f32" and var in ("3xtf32", "tf32bf16"):   # hi + lo / hi + bf16 [hi'|lo']: 8 bytes
        return 2 * (-(-K // 32) * 32) * 4 / K
    if dt == "f64" and var == "ozaki2":
        import json
        n = json.loads(pdl.query(f"ozaki2_plan/{K}"))["n"]
        kc = -(-K // 128) * 128
        return ((n + 1) * kc + 16) / K
    return 8 if dt == "f64" else 4


def model(M, N, K, tile, G, rate, es, t_meas=None, a_es=None):
    """Worst Worker's step: B column-panel all-gather (exposed), then its chunk
    launches in runtime.chunk_groups order, each starting when the previous one
    ends and its chunks have landed (broadcasts in chunk order, one chunk's bytes
    at a time at NVLINK), compute split over the chunks by rows."""
    from paper_conf_ipps_sandrieserbp11_b200 import runtime
    pdl.unload()
    pdl.load(pdl.descriptor_path(G))
    worst = 0.0
    for w in range(G):
        p = pdl.plan(M, N, K, tile, worker=w)
        wp = runtime.WorkerPlan(p["G"], p["Gr"], p["Gc"], p["r"], p["c"], p["row0"], p["row1"], p["col0"],
                                p["col1"], p["qa"], p["qb"], M, N, K)
        rows, cols = wp.rows, wp.cols
        t_comp = t_meas if t_meas is not None else 2.0 * rows * cols * K / rate
        t_b = K * cols * es * (1 - 1 / wp.Gr) / NVLINK                 # received B chunks
        chunk_t = wp.qa * K * (a_es or es) / NVLINK                     # one A chunk (raw or prepared)
        arrive, t = {}, 0.0
        for j in range(wp.Gc):                                          # broadcasts in chunk order
            if j != wp.c:
                t += chunk_t
            arrive[j] = 0.0 if j == wp.c else t
        now = 0.0
        for grp in runtime.chunk_groups(wp):
            if not grp:
                continue
            lo, hi = runtime.chunk_rows(wp, grp[0])[0], runtime.chunk_rows(wp, grp[-1])[1]
            now = max(now, max(arrive[j] for j in grp)) + t_comp * (hi - lo) / max(1, rows)
        worst = max(worst, t_b + now)
    pdl.unload()
    return worst


def main():
    r = rates()
    em = emulated()
    M = N = K = 16384
    rows = ["| variant | G=1 ms | G=2 | G=4 | G=8 | predicted S_8 | S_8 at the G=1 clock |",
            "|---|---|---|---|---|---|---|"]
    for key in CURRENT:   # variants measured only by the emulations: rate from their G = 1 step
        if key not in r and (*key, 1) in em:
            r[key] = 2.0 * M * N * K / em[(*key, 1)]
    for (dt, var), rate in sorted(r.items()):
        es = 8 if dt == "f64" else 4
        ts = [model(M, N, K, 1024, G, rate, es, em.get((dt, var, G)), a_bytes_per_elem(dt, var, K))
              for G in (1, 2, 4, 8)]
        src = "measured" if all((dt, var, G) in em for G in (1, 2, 4, 8)) else "rate"
        # power-capped variants run a short G = 8 step at a higher clock than the long
        # G = 1 step; scaling the G = 8 compute to the G = 1 clock removes that gain
        f1, f8 = CLOCK.get((dt, var, 1)), CLOCK.get((dt, var, 8))
        norm = "-"
        if f1 and f8 and (dt, var, 8) in em:
            t8c = em[(dt, var, 8)] * f8 / f1
            norm = f"{ts[0] / (ts[3] - em[(dt, var, 8)] + t8c):.2f} ({f1:.0f} / {f8:.0f} MHz)"
        rows.append(f"| {dt} {var} ({src}) | {ts[0] * 1e3:.1f} | {ts[1] * 1e3:.1f} | {ts[2] * 1e3:.1f} | "
                    f"{ts[3] * 1e3:.1f} | {ts[0] / ts[3]:.2f} | {norm} |")
    print("\n".join(rows))


if __name__ == "__main__":
    main()
