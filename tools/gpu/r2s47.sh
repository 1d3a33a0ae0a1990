# final evidence on the committed code: smoke, bench line, Ozaki-II ncu launch list + GEMM capture, reference arm, N=2 flow
mkdir -p gpurun_out
make -j8 all examples > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s47_smoke.txt 2>&1; echo smoke=$?
timeout 900 python bench.py > gpurun_out/r2s47_bench.json 2> gpurun_out/r2s47_bench.err; echo b=$?
timeout 900 python bench.py --gpus 2 --dist-backend gloo --config C3 --steps 3 > gpurun_out/r2s47_bench_n2.json 2> gpurun_out/r2s47_bench_n2.err; echo b2=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2s47_launches_oz2.csv python bench.py --variant ozaki2 --steps 1 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 > /dev/null 2>&1; echo ncu=$?
timeout 600 ncu --set full --clock-control none -k 'regex:oz2_(crt|row_bound|cert_cols)' -c 3 -o gpurun_out/prof_oz2aux_r23 -f python bench.py --variant ozaki2 --steps 1 --warmup 0 --no-alt --no-e2e --no-cpu-baseline --no-cublas --no-f32 > /dev/null 2>&1; echo ncu2=$?
