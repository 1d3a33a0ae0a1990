# final layout (16-wide bf16 pair blocks, BK 32 default, GROUP_M 8): full GPU suite + bench line + launch list + ncu of K2 mix
mkdir -p gpurun_out
make -j8 all examples > /dev/null
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2s22_tests.txt 2>&1; echo tests_rc=$?
tail -3 gpurun_out/r2s22_tests.txt
timeout 900 python bench.py > gpurun_out/r2s22_bench.json 2> gpurun_out/r2s22_bench.err; echo b=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2s22_launches_f32.csv python bench.py --dtype f32 --steps 2 --warmup 1 --no-alt --no-e2e --no-cpu-baseline --no-cublas > /dev/null 2>&1; echo ncu1=$?
timeout 600 ncu --set full --clock-control none --import-source on -k 'regex:gemm_3xtf32' -c 1 -o gpurun_out/prof_mix -f python bench.py --dtype f32 --steps 1 --warmup 0 --no-alt --no-cpu-baseline --no-cublas --no-e2e > /dev/null 2>&1; echo ncu2=$?
