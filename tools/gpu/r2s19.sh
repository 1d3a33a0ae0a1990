mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_tf32bf16.py tests/test_gpu_parity.py -q -x -k "not c4 and not c5" > gpurun_out/r2s19_tests.txt 2>&1; echo tests_rc=$?
tail -3 gpurun_out/r2s19_tests.txt
for v in tf32bf16 3xtf32; do for bk in 16 32; do
  PDL_K2_BK=$bk timeout 300 python bench.py --dtype f32 --variant $v --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e > gpurun_out/r2s19_${v}_bk$bk.json 2>/dev/null; echo ${v}_bk$bk=$?
done; done
