make -j8 all examples > /dev/null
python -m pytest tests/test_gpu_ozaki2.py -q -x > gpurun_out/r2s13_tests.txt 2>&1; echo tests_rc=$?
tail -3 gpurun_out/r2s13_tests.txt
ncu --set full --clock-control none -k 'regex:oz2?_gemm' -s 27 -c 1 -o gpurun_out/r2s13_prof_oz2cert -f python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-cublas --no-e2e --no-alt --no-f32 --variant ozaki2 > /dev/null 2>&1; echo ncu=$?
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2s13_launches_oz2.csv python bench.py --variant ozaki2 --steps 1 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 > /dev/null 2>&1; echo ncu2=$?
python bench.py --variant ozaki2 --steps 10 --warmup 3 --no-f32 --no-alt > gpurun_out/r2s13_bench_oz2.json 2> gpurun_out/r2s13_bench_oz2.err; echo b=$?
