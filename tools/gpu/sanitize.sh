# compute-sanitizer racecheck / synccheck / memcheck over the hand-written
# mbarrier / TMEM pipelines (K1, K2, K6 + certificate, the exchange path)
make -j8 all > /dev/null
CS=/usr/local/cuda/bin/compute-sanitizer
out=gpurun_out/r2_sanitize
mkdir -p $out
for tool in racecheck synccheck memcheck; do
  for spec in "dmma 1000 700 300" "3xtf32 1000 700 300" "ozaki2 777 1100 300" "ozaki2-flagged 600 530 260" "exchange 900 650 400 8"; do
    name=$(echo $spec | tr ' ' '_')
    extra=""
    [ $tool = racecheck ] && extra="--racecheck-report all"
    timeout 900 $CS --tool $tool $extra --kernel-name kns=pdlk --print-limit 50 python tools/sanitize_run.py $spec > $out/${tool}_${name}.txt 2>&1
    echo "$tool $name rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_${name}.txt | tail -2 | tr '\n' ' ')"
  done
done
