# R23 final form: full GPU suite, Ozaki-II timing with and without, sanitizers on the R23 paths
mkdir -p gpurun_out
make -j8 all examples > /dev/null
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r2s46_tests.txt 2>&1; echo tests_rc=$?; tail -2 gpurun_out/r2s46_tests.txt
for u in 1 0 1 0; do
  PDL_OZ2_CERT_UNIFORM=$u timeout 300 python bench.py --variant ozaki2 --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e --no-f32 > gpurun_out/r2s46_oz2_u$u.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/r2s46_oz2_u$u.json').read().strip().splitlines()[-1]); print($u, d['value'], d['ms_per_step'], d['clocks']['sm_mhz'])"
done
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in synccheck memcheck; do
  for spec in "ozaki2-uniform 777 1100 300" "ozaki2-mixed 777 1100 300" "ozaki2-mixed 300 200 260"; do
    name=${tool}_$(echo $spec | tr ' ' '_')
    timeout 900 $CS --tool $tool --kernel-name kns=pdlk --print-limit 50 python tools/sanitize_run.py $spec > gpurun_out/r2s46_$name.txt 2>&1
    echo "$name rc=$? $(grep -E 'ERROR SUMMARY|sanitize_run' gpurun_out/r2s46_$name.txt | tail -2 | tr '\n' ' ')"
  done
done
