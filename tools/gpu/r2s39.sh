# after R23: Ozaki-II per-Worker emulation (scaling model input) and the full bench line
mkdir -p gpurun_out
make -j8 all > /dev/null
timeout 1500 python tools/worker_emulate.py --dtype f64 --variant ozaki2 --sustain 1.5 > gpurun_out/r2s39_emulate_oz2.jsonl 2> gpurun_out/r2s39_emulate.err; echo em=$?
timeout 900 python bench.py > gpurun_out/r2s39_bench.json 2> gpurun_out/r2s39_bench.err; echo b=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2s39_launches_oz2.csv python bench.py --variant ozaki2 --steps 1 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 > /dev/null 2>&1; echo ncu=$?
