# tf32bf16 as the default FP32 variant: full GPU suite, per-Worker emulation, raster sweep, bench line
mkdir -p gpurun_out
make -j8 all examples > /dev/null
nvidia-smi -q -d POWER > gpurun_out/r2s17_power.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2s17_tests.txt 2>&1; echo tests_rc=$?
tail -3 gpurun_out/r2s17_tests.txt
for gm in 2 4 8 9 16; do
  PDL_GROUP_M=$gm timeout 300 python bench.py --dtype f32 --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e > gpurun_out/r2s17_gm$gm.json 2>/dev/null; echo gm$gm=$?
done
timeout 900 python tools/worker_emulate.py --dtype f32 --variant tf32bf16 --sustain 1.5 > gpurun_out/r2s17_emulate_f32_mix.jsonl 2> gpurun_out/r2s17_emulate.err; echo em=$?
timeout 900 python bench.py > gpurun_out/r2s17_bench.json 2> gpurun_out/r2s17_bench.err; echo b=$?
