mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_tf32bf16.py -q -x > gpurun_out/r2s34_tests.txt 2>&1; echo tests_rc=$?; tail -2 gpurun_out/r2s34_tests.txt
timeout 300 python bench.py --dtype f32 --variant 3xtf32 --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e > gpurun_out/r2s34_3x.json 2>/dev/null; echo b=$?
OUT=gpurun_out/r2s34 WHAT="k2x3" bash tools/profile.sh > gpurun_out/r2s34_profile.log 2>&1; echo prof=$?
