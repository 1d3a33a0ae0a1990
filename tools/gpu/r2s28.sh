mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for d in 0 5 0 5; do
  PDL_K2_DEBUG=$d timeout 300 python tools/k2_probe.py 16384 16384 16384 8192 8192 16384 >> gpurun_out/r2s28_probe.jsonl 2>&1; echo d$d=$?
done
cat gpurun_out/r2s28_probe.jsonl
