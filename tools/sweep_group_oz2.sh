#!/bin/bash
# raster group sweep for the Ozaki-II residue GEMMs (K6): step rate, clocks and
# DRAM bytes of one GEMM launch per setting
OUT=${OUT:-gpurun_out}
for g in 2 4 8 16 32 64; do
  r=$(PDL_GROUP_M=$g timeout 300 python bench.py --variant ozaki2 --steps 5 --warmup 3 --no-cpu-baseline --no-cublas --no-e2e --no-alt 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['kernel_ms'], d['clocks']['sm_mhz'])")
  PDL_GROUP_M=$g ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv -k regex:oz_gemm -s 14 -c 1 --log-file $OUT/sw_oz2_g$g.csv python bench.py --variant ozaki2 --steps 1 --warmup 1 --no-cpu-baseline --no-cublas --no-e2e --no-alt > /dev/null 2>&1
  b=$(python - "$OUT/sw_oz2_g$g.csv" <<'PY'
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
h = next(i for i, r in enumerate(rows) if "Metric Name" in r)
H = rows[h]
mi, ui, vi = H.index("Metric Name"), H.index("Metric Unit"), H.index("Metric Value")
sc = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
d = {r[mi]: float(r[vi].replace(",", "")) * sc.get(r[ui], 1) for r in rows[h + 1:] if len(r) > vi}
print(f"dram {(d.get('dram__bytes_read.sum', 0) + d.get('dram__bytes_write.sum', 0)) / 1e9:.2f} GB, {d.get('gpu__time_duration.sum', 0)} ")
PY
)
  echo "group_m=$g : $r : $b"
done
