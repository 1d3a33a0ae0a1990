mkdir -p gpurun_out
make -j8 all tools > /dev/null 2>&1
./tools/tc_microbench > gpurun_out/r2s18_tc_microbench.json; echo tc=$?
cat gpurun_out/r2s18_tc_microbench.json
for gm in 4 8; do
  PDL_GROUP_M=$gm timeout 300 python bench.py --dtype f32 --variant 3xtf32 --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e > gpurun_out/r2s18_3x_gm$gm.json 2>/dev/null; echo gm$gm=$?
done
