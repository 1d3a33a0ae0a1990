mkdir -p gpurun_out
make -j8 all > /dev/null
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:oz2_(residue_rows|split_cols_t|rowmax|colmax)' -c 4 --csv python bench.py --variant ozaki2 --steps 1 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 2>/dev/null | grep -i "gpu__time_duration" | awk -F'","' '{print substr($5,1,40), $NF}'
timeout 600 python -m pytest tests/test_gpu_ozaki2.py -q -x 2>&1 | tail -1
