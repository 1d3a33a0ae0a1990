# compute-sanitizer over the FP32 CTA-pair / 1-SM kernels of both FP32 variants (round 2, tf32bf16)
make -j8 all > /dev/null
CS=/usr/local/cuda/bin/compute-sanitizer
out=gpurun_out/r2s30_sanitize
mkdir -p $out
for tool in racecheck synccheck memcheck; do
  for cfg in "tf32bf16 2sm 32" "tf32bf16 2sm 16" "tf32bf16 1sm 32" "3xtf32 2sm 32" "3xtf32 2sm 16"; do set -- $cfg
    name=${tool}_$1_$2_bk$3
    extra=""
    [ $tool = racecheck ] && extra="--racecheck-report all"
    PDL_K2=$2 PDL_K2_BK=$3 timeout 900 $CS --tool $tool $extra --kernel-name kns=pdlk --print-limit 50 python tools/sanitize_run.py $1 1000 700 300 > $out/$name.txt 2>&1
    echo "$name rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize_run' $out/$name.txt | tail -2 | tr '\n' ' ')"
  done
done
