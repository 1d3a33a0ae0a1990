# tf32bf16 FP32 variant: correctness first, then timing against 3xtf32
mkdir -p gpurun_out
make -j8 all > /dev/null
timeout 900 python -m pytest tests/test_gpu_tf32bf16.py -q -x -m "gpu" > gpurun_out/r2s16_tests.txt 2>&1; echo tests_rc=$?
tail -5 gpurun_out/r2s16_tests.txt
for v in 3xtf32 tf32bf16; do
  PDL_SGEMM_VARIANT=$v timeout 300 python bench.py --dtype f32 --steps 10 --warmup 3 --no-alt --no-cpu-baseline --no-cublas > gpurun_out/r2s16_bench_$v.json 2> gpurun_out/r2s16_bench_$v.err; echo b_$v=$?
done
PDL_SGEMM_VARIANT=tf32bf16 timeout 300 ncu --set full --clock-control none -k 'regex:gemm_3xtf32' -c 1 -o gpurun_out/r2s16_prof_mix -f python bench.py --dtype f32 --steps 1 --warmup 0 --no-alt --no-cpu-baseline --no-cublas --no-e2e > /dev/null 2>&1; echo ncu=$?
