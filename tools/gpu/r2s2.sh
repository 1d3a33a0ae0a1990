make -j8 all examples > /dev/null
python -m pytest tests -m gpu -x -q > gpurun_out/r2s2_tests.txt 2>&1; echo tests_rc=$?
tail -5 gpurun_out/r2s2_tests.txt
