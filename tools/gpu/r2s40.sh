mkdir -p gpurun_out
make -j8 all > /dev/null
for occ in 3 2 3 2; do
  PDL_OZ2_CRT_OCC=$occ timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:oz2_crt -c 3 --csv python bench.py --variant ozaki2 --steps 2 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 2>/dev/null | grep -i "gpu__time_duration" | tail -1
done
