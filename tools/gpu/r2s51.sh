mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for pr in 256 128 0 256 128; do
  PDL_K2_L2PROMO=$pr timeout 300 python tools/k2_probe.py 16384 16384 16384 2>/dev/null | sed "s/^/promo=$pr /"
done
