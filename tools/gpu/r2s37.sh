# R23 sign-uniform certificate: Ozaki-II tests first, then the full suite, then timing
mkdir -p gpurun_out
make -j8 all examples > /dev/null
timeout 600 python -m pytest tests/test_gpu_ozaki2.py -q -x > gpurun_out/r2s37_oz_tests.txt 2>&1; echo oz_rc=$?
tail -15 gpurun_out/r2s37_oz_tests.txt
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r2s37_tests.txt 2>&1; echo tests_rc=$?
tail -5 gpurun_out/r2s37_tests.txt
for u in 1 0 1; do
  PDL_OZ2_CERT_UNIFORM=$u timeout 300 python bench.py --variant ozaki2 --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e --no-f32 > gpurun_out/r2s37_oz2_u$u.json 2>/dev/null; echo b_u$u=$?
  python -c "import json; d=json.loads(open('gpurun_out/r2s37_oz2_u$u.json').read().strip().splitlines()[-1]); print($u, d['value'], d['ms_per_step'], d['clocks']['sm_mhz'])"
done
