#!/bin/bash
# raster group sweep for the CTA-pair kernels (K2 v3, K4): kernel time per setting
# (PDL_GROUP_M overrides the compiled default of every CTA-pair kernel)
VARIANTS=${VARIANTS:-"--dtype f32|--variant ozaki|--dtype f32 --variant ozaki"}
IFS='|' read -ra VS <<< "$VARIANTS"
for g in ${GROUPS_M:-2 4 8 16 32}; do
  for v in "${VS[@]}"; do
    r=$(PDL_GROUP_M=$g timeout 300 python bench.py $v --steps 3 --warmup 2 --no-cpu-baseline --no-cublas --no-e2e --no-alt 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['kernel_ms'], d['clocks']['sm_mhz'])")
    echo "group_m=$g $v : $r"
  done
done
