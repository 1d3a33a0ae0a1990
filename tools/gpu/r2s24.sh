mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for v in tf32bf16 3xtf32; do for cfg in "2 32" "2 16" "4 32" "4 16"; do set -- $cfg
  PDL_K2_DEBUG=$1 PDL_K2_BK=$2 timeout 300 python bench.py --dtype f32 --variant $v --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e > gpurun_out/r2s24_${v}_d$1_bk$2.json 2>/dev/null; echo ${v}_d$1_bk$2=$?
done; done
