mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for pf in 0 2 4 8 16 0 4 8; do
  PDL_K2_PREFETCH=$pf timeout 300 python tools/k2_probe.py 16384 16384 16384 2>/dev/null | sed "s/^/pf=$pf /"
done
for pf in 0 8; do
  PDL_K2_PREFETCH=$pf PDL_K2_DEBUG=1 timeout 300 python tools/k2_probe.py 16384 16384 16384 2>/dev/null | sed "s/^/feedonly pf=$pf /"
done
