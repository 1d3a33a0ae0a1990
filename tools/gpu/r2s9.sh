make -j8 all examples > /dev/null
python -m pytest tests/test_gpu_multirank.py -q -x > gpurun_out/r2s9_tests.txt 2>&1; echo tests_rc=$?
tail -4 gpurun_out/r2s9_tests.txt
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --reps 5 > gpurun_out/r2s9_emulate_oz2_prepared.jsonl 2> gpurun_out/r2s9_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --reps 5 --raw > gpurun_out/r2s9_emulate_oz2_raw.jsonl 2>> gpurun_out/r2s9_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --reps 3 --gs 1,8 > gpurun_out/r2s9_emulate_f64.jsonl 2>> gpurun_out/r2s9_emulate.err; echo em=$?
