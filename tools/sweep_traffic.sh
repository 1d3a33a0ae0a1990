#!/bin/bash
# DRAM traffic / duration of the dominant kernels versus raster group (one ncu pass per setting)
P="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-cublas --no-e2e --no-alt"
m="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpc__cycles_elapsed.max.per_second"
for g in 4 8 16 32; do
  ncu --metrics $m --clock-control none -k regex:dgemm_k1 -s 1 -c 1 --csv env PDL_GROUP_M_K1=$g $P --dtype f64 2>/dev/null | grep -E "dram__|duration|cycles_elapsed" | awk -F'","' -v g=$g '{print "k1 g=" g, $(NF-2), $(NF-1), $NF}'
done
for g in 2 4 8; do
  ncu --metrics $m --clock-control none -k regex:gemm_3xtf32 -s 1 -c 1 --csv env PDL_GROUP_M=$g $P --dtype f32 2>/dev/null | grep -E "dram__|duration|cycles_elapsed" | awk -F'","' -v g=$g '{print "k2 g=" g, $(NF-2), $(NF-1), $NF}'
  ncu --metrics $m --clock-control none -k regex:oz_gemm -s 6 -c 1 --csv env PDL_GROUP_M=$g $P --variant ozaki 2>/dev/null | grep -E "dram__|duration|cycles_elapsed" | awk -F'","' -v g=$g '{print "oz g=" g, $(NF-2), $(NF-1), $NF}'
done
