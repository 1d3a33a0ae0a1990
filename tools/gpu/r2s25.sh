mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for d in 4 0; do
  PDL_K2_DEBUG=$d timeout 300 python tools/k2_probe.py 16384 16384 16384 9472 9472 65536 18944 18944 8192 4096 4096 65536 >> gpurun_out/r2s25_probe.jsonl 2>&1; echo d$d=$?
done
cat gpurun_out/r2s25_probe.jsonl
