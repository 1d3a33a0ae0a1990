# compute-sanitizer over the R23 paths (certificate skip, CRT certificate, per-lane column bits)
make -j8 all > /dev/null
CS=/usr/local/cuda/bin/compute-sanitizer
out=gpurun_out/r2s38_sanitize
mkdir -p $out
for tool in synccheck racecheck memcheck; do
  for spec in "ozaki2-uniform 777 1100 300" "ozaki2-mixed 777 1100 300" "ozaki2-mixed 300 200 260"; do
    name=${tool}_$(echo $spec | tr ' ' '_')
    extra=""
    [ $tool = racecheck ] && extra="--racecheck-report all"
    timeout 900 $CS --tool $tool $extra --kernel-name kns=pdlk --print-limit 50 python tools/sanitize_run.py $spec > $out/$name.txt 2>&1
    echo "$name rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize_run' $out/$name.txt | tail -2 | tr '\n' ' ')"
  done
done
