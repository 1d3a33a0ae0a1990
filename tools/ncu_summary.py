"""Summarise ncu --set full captures (.ncu-rep) into profiles/ (run here, no GPU).

    python tools/ncu_summary.py ROUND gpurun_out/prof_k1.ncu-rep [...]

Writes profiles/<ROUND>_ncu_<name>.json with the metrics the roofline and the
judge use (duration, DRAM bytes, pipe utilisation, L2 / L1 throughput, stall
reasons) and updates profiles/ncu_traffic.json (DRAM bytes per launch by
dtype/config) which bench.py reports as roofline.traffic.
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_tensor_subpipe_hmma.avg.pct_of_peak_sustained_active",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_tc_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "gpc__cycles_elapsed.max.per_second", "smsp__inst_executed.sum",
]


def raw(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True,
                                  stderr=subprocess.DEVNULL)
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def summarise(rep):
    hdr, units, rows = raw(rep)
    res = []
    for r in rows:
        d = {"kernel": r[hdr.index("Kernel Name")][:80]}
        for k in KEYS:
            if k in hdr:
                v = r[hdr.index(k)].replace(",", "")
                try:
                    d[k] = float(v)
                except ValueError:
                    d[k] = v
                u = units[hdr.index(k)]
                if u:
                    d[k + " [unit]"] = u
        stalls = {}
        for i, h in enumerate(hdr):
            if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued"):
                try:
                    stalls[h.replace("smsp__pcsamp_warps_issue_stalled_", "")] = float(r[i].replace(",", ""))
                except ValueError:
                    pass
        tot = sum(stalls.values()) or 1.0
        d["stall_share"] = {k: round(v / tot, 4) for k, v in sorted(stalls.items(), key=lambda x: -x[1])[:8]}
        res.append(d)
    return res


def to_bytes(v, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    return v * scale.get(unit, 1)


def main():
    rnd = sys.argv[1]
    traffic_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        traffic = json.load(open(traffic_path))
    except (OSError, ValueError):
        traffic = {}
    for rep in sys.argv[2:]:
        name = os.path.splitext(os.path.basename(rep))[0]
        s = summarise(rep)
        with open(os.path.join(ROOT, "profiles", f"{rnd}_ncu_{name}.json"), "w") as f:
            json.dump(s, f, indent=1)
        for d in s:
            rd = to_bytes(d.get("dram__bytes_read.sum", 0), d.get("dram__bytes_read.sum [unit]", "byte"))
            wr = to_bytes(d.get("dram__bytes_write.sum", 0), d.get("dram__bytes_write.sum [unit]", "byte"))
            key = None   # only the bench's dominant-kernel captures (not e.g. the Ozaki-II recompute K1)
            if "dgemm_k1" in d["kernel"] and name.startswith("prof_k1"):
                key = "f64/C4"
            elif "gemm_3xtf32" in d["kernel"] and name.startswith("prof_k2x3"):
                key = "f32/C4"                      # 3xtf32 (bench's f32_3xtf32 leg)
            elif "gemm_3xtf32" in d["kernel"] and (name.startswith("prof_k2") or name.startswith("prof_mix")):
                key = "f32_tf32bf16/C4"             # the FP32 default
            if key:
                traffic[key] = int(rd + wr)
            print(name, d["kernel"][:40], "dram bytes", int(rd + wr), d.get("stall_share"))
    with open(traffic_path, "w") as f:
        json.dump(traffic, f, indent=1)


if __name__ == "__main__":
    main()
