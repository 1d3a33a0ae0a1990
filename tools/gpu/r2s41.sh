mkdir -p gpurun_out
make -j8 all > /dev/null
for u in 1 0; do
  PDL_OZ2_CERT_UNIFORM=$u timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:oz2_crt -c 2 --csv python bench.py --variant ozaki2 --steps 2 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 2>/dev/null | grep -i "gpu__time_duration" | tail -1 | awk -F'","' '{print $5, $NF}'
done
timeout 600 python -m pytest tests/test_gpu_ozaki2.py -q -x -k "uniform or mixed or certificate" 2>&1 | tail -2
