mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
python tools/h2d_probe.py > gpurun_out/r2s23_h2d.json 2>&1; echo h2d=$?; cat gpurun_out/r2s23_h2d.json
for rc in "8 4" "4 4" "8 2" "16 4" "8 8"; do set -- $rc
  PDL_PIPE_RB=$1 PDL_PIPE_CP=$2 timeout 300 python bench.py --dtype f32 --steps 5 --warmup 3 --no-alt --no-cpu-baseline --no-cublas > gpurun_out/r2s23_e2e_$1_$2.json 2>/dev/null; echo e2e_$1_$2=$?
done
timeout 900 python tools/worker_emulate.py --dtype f32 --variant tf32bf16 --sustain 1.5 > gpurun_out/r2s23_emulate_f32_mix.jsonl 2> gpurun_out/r2s23_emulate.err; echo em=$?
