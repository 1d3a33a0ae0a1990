make -j8 all examples > /dev/null
python -m pytest tests -m gpu -q > gpurun_out/r2s3_tests.txt 2>&1; echo tests_rc=$?
tail -15 gpurun_out/r2s3_tests.txt
