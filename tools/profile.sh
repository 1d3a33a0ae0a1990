#!/bin/bash
# ncu evidence for the dominant kernels (run on the GPU box via gpurun).
# 1) launch list (gpu__time_duration, one pass, no replay) of the bench commands
# 2) one --set full capture per dominant kernel at the bench's launch configuration (C4)
set -x
OUT=${OUT:-gpurun_out}
WHAT=${WHAT:-"k1 k2 k3 oz"}
mkdir -p $OUT
B="python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-cublas --no-alt --e2e-steps 1"
P="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-cublas --no-e2e --no-alt"
for w in $WHAT; do
  case $w in
    k1) ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_f64.csv $B --dtype f64 > $OUT/launches_f64.log 2>&1
        ncu --set full --clock-control none --import-source on -k regex:dgemm_k1 -s 1 -c 1 -o $OUT/prof_k1 -f $P --dtype f64 > $OUT/prof_k1.log 2>&1 ;;
    k2) ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_f32.csv $B --dtype f32 > $OUT/launches_f32.log 2>&1
        ncu --set full --clock-control none --import-source on -k regex:gemm_3xtf32 -s 1 -c 1 -o $OUT/prof_k2 -f $P --dtype f32 > $OUT/prof_k2.log 2>&1 ;;
    k3) ncu --set full --clock-control none --import-source on -k regex:split -s 2 -c 2 -o $OUT/prof_k3 -f $P --dtype f32 > $OUT/prof_k3.log 2>&1 ;;
    oz) ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_oz.csv $B --variant ozaki > $OUT/launches_oz.log 2>&1
        ncu --set full --clock-control none --import-source on -k regex:oz_gemm -s 7 -c 1 -o $OUT/prof_oz -f $P --variant ozaki > $OUT/prof_oz.log 2>&1
        ncu --set full --clock-control none --import-source on -k regex:oz_split -s 2 -c 2 -o $OUT/prof_ozsplit -f $P --variant ozaki > $OUT/prof_ozsplit.log 2>&1 ;;
  esac
done
ls -la $OUT
