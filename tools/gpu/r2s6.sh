make -j8 all examples > /dev/null
python -m pytest tests/test_gpu_multirank.py tests/test_gpu_fullsize.py -q -k "prepared or prep_a or late or missing or integer or distributed" > gpurun_out/r2s6_tests.txt 2>&1; echo tests_rc=$?
tail -6 gpurun_out/r2s6_tests.txt
python tools/worker_emulate.py --dtype f32 --reps 3 > gpurun_out/r2s6_emulate_f32_prepared.jsonl 2> gpurun_out/r2s6_emulate.err; echo em1=$?
python tools/worker_emulate.py --dtype f32 --reps 3 --raw > gpurun_out/r2s6_emulate_f32_raw.jsonl 2>> gpurun_out/r2s6_emulate.err; echo em2=$?
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --reps 3 > gpurun_out/r2s6_emulate_oz2.jsonl 2>> gpurun_out/r2s6_emulate.err; echo em3=$?
bash tools/gpu/sanitize.sh
