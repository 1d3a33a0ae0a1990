"""Regenerate the per-Worker compute table and the S_8 table of DESIGN.md section 7
and profiles/r02_scaling_model.md from profiles/r02_worker_emulate_*.jsonl and
tools/scaling_model.py (no GPU)."""
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ROWS = (("f64", "FP64 K1 DMMA (raw)"),
        ("f32_tf32bf16", "FP32 tf32bf16, the FP32 default (prepared TF32 hi + BF16 pairs)"),
        ("f32", "FP32 3xTF32 (prepared TF32 hi/lo)"),
        ("f64_ozaki2", "FP64 Ozaki-II + certificate (prepared residues)"))


def emulate_table():
    rows = ["| variant (A exchange) | G=1 ms | G=2 | G=4 | G=8 | G=8 speedup | SM MHz G=1 / G=8 |",
            "|---|---|---|---|---|---|---|"]
    for fn, lab in ROWS:
        d = {}
        with open(os.path.join(ROOT, "profiles", f"r02_worker_emulate_{fn}.jsonl")) as f:
            for line in f:
                j = json.loads(line)
                if j.get("config") == "C4" and "G" in j:
                    d[j["G"]] = j
        t = [d[g]["max_concurrent_ms"] for g in (1, 2, 4, 8)]
        rows.append(f"| {lab} | " + " | ".join(f"{x:.2f}" for x in t) +
                    f" | {t[0] / t[3]:.2f} | {d[1].get('sm_mhz_worst'):.0f} / {d[8].get('sm_mhz_worst'):.0f} |")
    return "\n".join(rows)


def replace_table(text, anchor, table):
    i = text.index(anchor) + len(anchor)
    j = text.index("\n|", i) + 1          # first table line after the anchor
    k = j
    while k < len(text) and text[k] == "|":
        k = text.index("\n", k) + 1
    return text[:j] + table + "\n" + text[k:]


def main():
    em = emulate_table()
    sc = subprocess.check_output([sys.executable, os.path.join(ROOT, "tools", "scaling_model.py")], text=True).strip()
    p = os.path.join(ROOT, "DESIGN.md")
    s = open(p).read()
    s = replace_table(s, "Worker position of a grid row", em)
    s = replace_table(s, "scaled to the G = 1 clock (`profiles/r02_scaling_model.md`):", sc)
    open(p, "w").write(s)
    m = os.path.join(ROOT, "profiles", "r02_scaling_model.md")
    t = open(m).read()
    t = replace_table(t, "Per-Worker compute (ms, worst Worker):", em)
    t = replace_table(t, "Modelled step (ms) and S_8:", sc)
    open(m, "w").write(t)
    print(em)
    print(sc)


if __name__ == "__main__":
    main()
