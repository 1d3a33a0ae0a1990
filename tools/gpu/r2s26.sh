mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for sms in 0 72 40; do for d in 1 4 0; do
  PROBE_SMS=$sms PDL_K2_DEBUG=$d timeout 300 python tools/k2_probe.py 8192 8192 16384 >> gpurun_out/r2s26_probe.jsonl 2>&1; echo s${sms}_d$d=$?
done; done
cat gpurun_out/r2s26_probe.jsonl
