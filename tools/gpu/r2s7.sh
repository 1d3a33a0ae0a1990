make -j8 all examples > /dev/null
for i in 1 2; do
python tools/worker_emulate.py --dtype f32 --reps 5 > gpurun_out/r2s7_emulate_f32_prepared_$i.jsonl 2>> gpurun_out/r2s7_emulate.err; echo em1=$?
python tools/worker_emulate.py --dtype f32 --reps 5 --raw > gpurun_out/r2s7_emulate_f32_raw_$i.jsonl 2>> gpurun_out/r2s7_emulate.err; echo em2=$?
done
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --reps 5 > gpurun_out/r2s7_emulate_oz2.jsonl 2>> gpurun_out/r2s7_emulate.err; echo em3=$?
PDL_K2=2sm timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --racecheck-report all --kernel-name kns=pdlk --print-limit 20 python tools/sanitize_run.py 3xtf32 1000 700 300 > gpurun_out/r2_sanitize/racecheck_3xtf32_2sm_1000_700_300.txt 2>&1; echo rc_k2=$?
tail -3 gpurun_out/r2_sanitize/racecheck_3xtf32_2sm_1000_700_300.txt
PDL_OZ2_PERSIST=0 timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --racecheck-report all --kernel-name kns=pdlk --print-limit 20 python tools/sanitize_run.py ozaki2 777 1100 300 > gpurun_out/r2_sanitize/racecheck_ozaki2_nonpersistent_777_1100_300.txt 2>&1; echo rc_oz=$?
tail -3 gpurun_out/r2_sanitize/racecheck_ozaki2_nonpersistent_777_1100_300.txt
