mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for gm in 16 8 32 4 16; do
  PDL_GROUP_M=$gm timeout 300 python bench.py --variant ozaki2 --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e --no-f32 > gpurun_out/r2s35_gm$gm.json 2>/dev/null; echo gm$gm=$?
  python -c "import json; d=json.loads(open('gpurun_out/r2s35_gm$gm.json').read().strip().splitlines()[-1]); print($gm, d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['clocks'].get('power_w'))"
done
