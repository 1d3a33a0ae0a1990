make -j8 all examples > /dev/null
python tools/worker_emulate.py --dtype f32 --sustain 1.5 > gpurun_out/r2s14_emulate_f32.jsonl 2> gpurun_out/r2s14_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --sustain 1.5 > gpurun_out/r2s14_emulate_oz2.jsonl 2>> gpurun_out/r2s14_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --sustain 1.0 > gpurun_out/r2s14_emulate_f64.jsonl 2>> gpurun_out/r2s14_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f32 --sustain 1.5 --raw --gs 1,8 > gpurun_out/r2s14_emulate_f32_raw.jsonl 2>> gpurun_out/r2s14_emulate.err; echo em=$?
python tools/worker_emulate.py --dtype f64 --variant ozaki2 --sustain 1.5 --raw --gs 1,8 > gpurun_out/r2s14_emulate_oz2_raw.jsonl 2>> gpurun_out/r2s14_emulate.err; echo em=$?
