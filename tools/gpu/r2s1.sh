# round-2 GPU session 1: full GPU suite + benches
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
make -j8 all examples > /dev/null
python -m pytest tests -m gpu -x -q > gpurun_out/r2s1_tests.txt 2>&1; echo tests_rc=$?
tail -5 gpurun_out/r2s1_tests.txt
python bench.py --steps 5 --warmup 3 > gpurun_out/r2s1_bench.json 2> gpurun_out/r2s1_bench.err; echo bench_rc=$?
python bench.py --gpus 2 --config C3 --steps 3 --warmup 3 --cpu-seconds 3 > gpurun_out/r2s1_bench_n2.json 2> gpurun_out/r2s1_bench_n2.err; echo bench2_rc=$?
