mkdir -p gpurun_out
make -j8 all examples > /dev/null
timeout 600 python -m pytest tests/test_gpu_ozaki2.py tests/test_gpu_exchange.py tests/test_gpu_multirank.py -q -x > gpurun_out/r2s42_tests.txt 2>&1; echo tests_rc=$?; tail -3 gpurun_out/r2s42_tests.txt
for u in 1 0 1 0; do
  PDL_OZ2_CERT_UNIFORM=$u timeout 300 python bench.py --variant ozaki2 --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e --no-f32 > gpurun_out/r2s42_oz2_u$u.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/r2s42_oz2_u$u.json').read().strip().splitlines()[-1]); print($u, d['value'], d['ms_per_step'], d['clocks']['sm_mhz'])"
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:oz2_(crt|cert)' -c 4 --csv python bench.py --variant ozaki2 --steps 2 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 2>/dev/null | grep -i "gpu__time_duration" | awk -F'","' '{print $5, $NF}'
