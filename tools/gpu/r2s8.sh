make -j8 all examples > /dev/null
mkdir -p gpurun_out/r2_sanitize
python -m pytest tests -m gpu -q > gpurun_out/r2s8_tests.txt 2>&1; echo tests_rc=$?
tail -4 gpurun_out/r2s8_tests.txt
python bench.py --steps 10 --warmup 3 > gpurun_out/r2s8_bench.json 2> gpurun_out/r2s8_bench.err; echo bench_rc=$?
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2s8_launches_oz2.csv python bench.py --variant ozaki2 --steps 1 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 > /dev/null 2>&1; echo ncu_rc=$?
PDL_K2=2sm timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --racecheck-report all --kernel-name kns=pdlk --print-limit 20 python tools/sanitize_run.py 3xtf32 1000 700 300 > gpurun_out/r2_sanitize/racecheck_3xtf32_2sm_1000_700_300.txt 2>&1; echo rc_k2=$?
tail -2 gpurun_out/r2_sanitize/racecheck_3xtf32_2sm_1000_700_300.txt
PDL_OZ2_PERSIST=0 timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --racecheck-report all --kernel-name kns=pdlk --print-limit 20 python tools/sanitize_run.py ozaki2 777 1100 300 > gpurun_out/r2_sanitize/racecheck_ozaki2_nonpersistent_777_1100_300.txt 2>&1; echo rc_oz=$?
tail -2 gpurun_out/r2_sanitize/racecheck_ozaki2_nonpersistent_777_1100_300.txt
