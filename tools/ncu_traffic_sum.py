"""DRAM bytes of one bench step of a multi-launch task variant (run here, no GPU).

    python tools/ncu_traffic_sum.py gpurun_out/traffic_ozaki.csv ozaki/C4 [...]

Each CSV is an `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,...
--csv --log-file` capture of the GEMM launches of one step (tools/profile.sh).
The per-step sum (all slice-diagonal / residue GEMM launches, which bench.py's
roofline "achieved" also spans) is written to profiles/ncu_traffic.json under
the given key, which bench.py reports as roofline.traffic.
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def step_bytes(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Metric Name" in r)
    H = rows[h]
    mi, ui, vi = H.index("Metric Name"), H.index("Metric Unit"), H.index("Metric Value")
    tot, n = 0.0, 0
    for r in rows[h + 1:]:
        if len(r) > vi and r[mi] in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            tot += float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1)
            n += r[mi] == "dram__bytes_read.sum"
    return int(tot), n


def main():
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    traffic = json.load(open(tp)) if os.path.exists(tp) else {}
    args = sys.argv[1:]
    for path, key in zip(args[::2], args[1::2]):
        b, n = step_bytes(path)
        traffic[key] = b
        print(f"{key}: {b / 1e9:.2f} GB over {n} launches")
    json.dump(traffic, open(tp, "w"), indent=1)


if __name__ == "__main__":
    main()
