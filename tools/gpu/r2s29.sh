# e2e pipeline fill: smaller first row band / column panel (FP64 C4 through the C ABI on pinned host operands)
mkdir -p gpurun_out
make -j8 all > /dev/null 2>&1
run() { tag=$1; shift; env "$@" timeout 600 python bench.py --steps 4 --warmup 3 --no-alt --no-cpu-baseline --no-cublas --no-f32 > gpurun_out/r2s29_$tag.json 2>/dev/null; echo $tag=$?; }
run base
run f2c2 PDL_PIPE_FIRST=2 PDL_PIPE_FIRST_COL=2
run f4c4 PDL_PIPE_FIRST=4 PDL_PIPE_FIRST_COL=4
run c4 PDL_PIPE_FIRST_COL=4
run rb8cp8f2 PDL_PIPE_RB=8 PDL_PIPE_CP=8 PDL_PIPE_FIRST=2 PDL_PIPE_FIRST_COL=2
run rb16cp8f2 PDL_PIPE_RB=16 PDL_PIPE_CP=8 PDL_PIPE_FIRST=2 PDL_PIPE_FIRST_COL=2
