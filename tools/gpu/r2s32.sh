# round-2 final validation on the committed code: smoke, full GPU suite, bench line, reference arm, N=2 flow
mkdir -p gpurun_out
make -j8 all examples > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s32_smoke.txt 2>&1; echo smoke=$?
timeout 2700 python -m pytest tests -m gpu -q > gpurun_out/r2s32_tests.txt 2>&1; echo tests_rc=$?
tail -3 gpurun_out/r2s32_tests.txt
timeout 900 python bench.py > gpurun_out/r2s32_bench.json 2> gpurun_out/r2s32_bench.err; echo b=$?
timeout 900 python bench.py --gpus 2 --dist-backend gloo --config C3 --steps 3 > gpurun_out/r2s32_bench_n2.json 2> gpurun_out/r2s32_bench_n2.err; echo b2=$?
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r2s32_bench_ref.json 2> gpurun_out/r2s32_bench_ref.err; echo bref=$?
