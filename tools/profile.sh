#!/bin/bash
# ncu evidence for the dominant kernels (run on the GPU box via gpurun).
# 1) launch list (gpu__time_duration, one pass, no replay) of the bench commands
# 2) one --set full capture per dominant kernel at the bench's launch configuration (C4)
# 3) DRAM bytes of every GEMM launch of one step of the multi-launch variants (the
#    roofline "traffic" of a step: tools/ncu_traffic_sum.py)
set -x
OUT=${OUT:-gpurun_out}
WHAT=${WHAT:-"k1 k2 k2x3 k3 oz2"}   # k2: the FP32 default (tf32bf16), k2x3: 3xtf32
mkdir -p $OUT
B="python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-cublas --no-alt --e2e-steps 1"
P="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-cublas --no-e2e --no-alt"
DR="--metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv"
for w in $WHAT; do
  case $w in
    k1) ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_f64.csv $B --dtype f64 > $OUT/launches_f64.log 2>&1
        ncu --set full --clock-control none --import-source on -k regex:dgemm_k1 -s 1 -c 1 -o $OUT/prof_k1 -f $P --dtype f64 > $OUT/prof_k1.log 2>&1 ;;
    k2) ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_f32.csv $B --dtype f32 > $OUT/launches_f32.log 2>&1
        ncu --set full --clock-control none --import-source on -k regex:gemm_3xtf32 -s 1 -c 1 -o $OUT/prof_k2 -f $P --dtype f32 > $OUT/prof_k2.log 2>&1 ;;
    k2x3) ncu --set full --clock-control none --import-source on -k regex:gemm_3xtf32 -s 1 -c 1 -o $OUT/prof_k2x3 -f $P --dtype f32 --variant 3xtf32 > $OUT/prof_k2x3.log 2>&1 ;;
    k3) ncu --set full --clock-control none --import-source on -k regex:split -s 2 -c 2 -o $OUT/prof_k3 -f $P --dtype f32 > $OUT/prof_k3.log 2>&1 ;;
    oz2) ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_oz2.csv $B --variant ozaki2 > $OUT/launches_oz2.log 2>&1
        # 14 GEMM launches per step at C4 (13 moduli + the certificate, R21); step 2 of the
        # warm-up + timed run: skip the first step's 14, capture a residue GEMM and the certificate
        ncu --set full --clock-control none --import-source on -k 'regex:oz2?_gemm' -s 14 -c 1 -o $OUT/prof_oz2 -f $P --variant ozaki2 > $OUT/prof_oz2.log 2>&1
        ncu --set full --clock-control none --import-source on -k 'regex:oz2?_gemm' -s 27 -c 1 -o $OUT/prof_oz2cert -f $P --variant ozaki2 > $OUT/prof_oz2cert.log 2>&1
        ncu --set full --clock-control none --import-source on -k 'regex:oz2_(rowmax|residue|colmax|split|crt|reconstruct)|dgemm_k1' -s 6 -c 6 -o $OUT/prof_oz2aux -f $P --variant ozaki2 > $OUT/prof_oz2aux.log 2>&1
        ncu $DR -k 'regex:oz2?_gemm' -s 14 -c 14 --log-file $OUT/traffic_ozaki2.csv $P --variant ozaki2 > $OUT/traffic_oz2.log 2>&1 ;;
  esac
done
ls -la $OUT
