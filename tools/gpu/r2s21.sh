mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
for v in tf32bf16; do for d in 2 3; do
  PDL_K2_DEBUG=$d timeout 300 python bench.py --dtype f32 --variant $v --steps 8 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-e2e > gpurun_out/r2s21_${v}_d$d.json 2>/dev/null; echo ${v}_d$d=$?
done; done
