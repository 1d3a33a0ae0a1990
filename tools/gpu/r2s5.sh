make -j8 all examples > /dev/null
python -m pytest tests -m gpu -q > gpurun_out/r2s5_tests.txt 2>&1; echo tests_rc=$?
tail -6 gpurun_out/r2s5_tests.txt
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2s5_launches_oz2.csv python bench.py --variant ozaki2 --steps 1 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 > /dev/null 2>&1; echo ncu_rc=$?
bash tools/gpu/sanitize.sh
