make -j8 all examples > /dev/null
python -m pytest tests/test_gpu_ozaki2.py tests/test_gpu_fullsize.py tests/test_gpu_multirank.py -q -x > gpurun_out/r2s12_tests.txt 2>&1; echo tests_rc=$?
tail -4 gpurun_out/r2s12_tests.txt
ncu --set full --clock-control none -k 'regex:oz2?_gemm' -s 27 -c 1 -o gpurun_out/r2s12_prof_oz2cert -f python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-cublas --no-e2e --no-alt --no-f32 --variant ozaki2 > /dev/null 2>&1; echo ncu=$?
python bench.py --variant ozaki2 --steps 10 --warmup 3 --no-f32 --no-alt > gpurun_out/r2s12_bench_oz2.json 2> gpurun_out/r2s12_bench_oz2.err; echo b=$?
python tools/worker_emulate.py --dtype f32 --reps 5 > gpurun_out/r2s12_emulate_f32.jsonl 2> gpurun_out/r2s12_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --reps 5 > gpurun_out/r2s12_emulate_oz2.jsonl 2>> gpurun_out/r2s12_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --reps 3 > gpurun_out/r2s12_emulate_f64.jsonl 2>> gpurun_out/r2s12_emulate.err; echo em=$?
