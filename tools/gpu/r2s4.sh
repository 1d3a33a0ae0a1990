make -j8 all examples > /dev/null
python -m pytest tests/test_gpu_ozaki2.py tests/test_gpu_ozaki_retired.py -q -x > gpurun_out/r2s4_oz2.txt 2>&1; echo oz2_rc=$?
tail -25 gpurun_out/r2s4_oz2.txt
python -m pytest tests -m gpu -q > gpurun_out/r2s4_tests.txt 2>&1; echo tests_rc=$?
tail -15 gpurun_out/r2s4_tests.txt
python bench.py --steps 5 --warmup 3 --no-f32 --no-e2e --no-cpu-baseline > gpurun_out/r2s4_bench.json 2> gpurun_out/r2s4_bench.err; echo bench_rc=$?
