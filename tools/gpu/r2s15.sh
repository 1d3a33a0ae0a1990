# round 2, session 2: full GPU suite, smoke, default bench line, N=2 flow
mkdir -p gpurun_out
make -j8 all examples > /dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/r2s15_smi.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s15_smoke.txt 2>&1; echo smoke=$?
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2s15_tests.txt 2>&1; echo tests_rc=$?
tail -3 gpurun_out/r2s15_tests.txt
python bench.py > gpurun_out/r2s15_bench.json 2> gpurun_out/r2s15_bench.err; echo b=$?
python bench.py --gpus 2 --dist-backend gloo --config C3 --steps 3 > gpurun_out/r2s15_bench_n2.json 2> gpurun_out/r2s15_bench_n2.err; echo b2=$?
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r2s15_bench_ref.json 2> gpurun_out/r2s15_bench_ref.err; echo bref=$?
