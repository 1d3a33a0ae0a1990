mkdir -p gpurun_out
make -j8 all > /dev/null
timeout 600 python -m pytest tests/test_gpu_ozaki2.py -q -x > gpurun_out/r2s45_tests.txt 2>&1; echo tests_rc=$?; tail -2 gpurun_out/r2s45_tests.txt
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none -k 'regex:oz2_crt' -c 2 --csv python bench.py --variant ozaki2 --steps 2 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 2>/dev/null | grep -i "gpu__time_duration\|dram__bytes" | awk -F'","' '{print $5, $(NF-2), $NF}'
