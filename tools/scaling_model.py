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
CURRENT = {("f64", "dmma"), ("f32", "3xtf32"), ("f64", "ozaki2")}


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
        if (fn.startswith("r01_worker_emulate_") or fn.startswith("r02_worker_emulate_")) and fn.endswith(".jsonl"):
            with open(os.path.join(ROOT, "profiles", fn)) as f:
                for line in f:
                    d = json.loads(line)
                    if "G" in d and d.get("config") == "C4":
                        var = {"default": "dmma" if d["dtype"] == "f64" else "3xtf32"}.get(
                            d.get("variant", "default"), d.get("variant"))
                        out[(d["dtype"], var, d["G"])] = d["max_concurrent_ms"] / 1e3
    return out


def a_bytes_per_elem(dt, var, K):
    """Bytes per A element on NVLink: FP32 3xTF32 exchanges prepared TF32 hi/lo rows
    (runtime.PanelBuffers prep_bytes: 2 Kp floats per row), the others raw rows."""
    if dt == "f32" and var == "3xtf32":
        return 2 * (-(-K // 32) * 32) * 4 / K
    return 8 if dt == "f64" else 4


def model(M, N, K, tile, G, rate, es, t_meas=None, a_es=None):
    pdl.unload()
    pdl.load(pdl.descriptor_path(G))
    worst = 0.0
    for w in range(G):
        p = pdl.plan(M, N, K, tile, worker=w)
        rows, cols = p["row1"] - p["row0"], p["col1"] - p["col0"]
        t_comp = t_meas if t_meas is not None else 2.0 * rows * cols * K / rate
        b_bytes = K * cols * es * (1 - 1 / p["Gr"])            # received B chunks
        a_chunk = p["qa"] * K * (a_es or es)                    # one A chunk (raw or prepared)
        t_b = b_bytes / NVLINK
        # the own chunk (1/Gc of the work) computes while the other Gc-1 chunks arrive
        t_own = t_comp / p["Gc"]
        t_a_exposed = max(0.0, (p["Gc"] - 1) * a_chunk / NVLINK - t_own)
        worst = max(worst, t_b + t_a_exposed + t_comp)
    pdl.unload()
    return worst


def main():
    r = rates()
    em = emulated()
    M = N = K = 16384
    rows = ["| variant | G=1 ms | G=2 | G=4 | G=8 | predicted S_8 |", "|---|---|---|---|---|---|"]
    for (dt, var), rate in sorted(r.items()):
        es = 8 if dt == "f64" else 4
        ts = [model(M, N, K, 1024, G, rate, es, em.get((dt, var, G)), a_bytes_per_elem(dt, var, K))
              for G in (1, 2, 4, 8)]
        src = "measured" if all((dt, var, G) in em for G in (1, 2, 4, 8)) else "rate"
        rows.append(f"| {dt} {var} ({src}) | {ts[0] * 1e3:.1f} | {ts[1] * 1e3:.1f} | {ts[2] * 1e3:.1f} | "
                    f"{ts[3] * 1e3:.1f} | {ts[0] / ts[3]:.2f} |")
    print("\n".join(rows))


if __name__ == "__main__":
    main()
