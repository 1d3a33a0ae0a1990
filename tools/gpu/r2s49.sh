# final: smoke, full GPU suite, bench line on the final code
mkdir -p gpurun_out
make -j8 all examples > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s49_smoke.txt 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2s49_tests.txt 2>&1; echo tests_rc=$?; tail -2 gpurun_out/r2s49_tests.txt
timeout 900 python bench.py > gpurun_out/r2s49_bench.json 2> gpurun_out/r2s49_bench.err; echo b=$?
