make -j8 all examples > /dev/null
python tools/worker_emulate.py --dtype f32 --reps 5 > gpurun_out/r2s10_emulate_f32.jsonl 2> gpurun_out/r2s10_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --reps 5 > gpurun_out/r2s10_emulate_oz2.jsonl 2>> gpurun_out/r2s10_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --reps 3 > gpurun_out/r2s10_emulate_f64.jsonl 2>> gpurun_out/r2s10_emulate.err; echo em=$?
python -m pytest tests -m gpu -q > gpurun_out/r2s10_tests.txt 2>&1; echo tests_rc=$?
tail -4 gpurun_out/r2s10_tests.txt
