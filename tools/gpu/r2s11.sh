make -j8 all examples > /dev/null
OUT=gpurun_out/r2prof WHAT="k1 k2 oz2" bash tools/profile.sh > gpurun_out/r2s11_profile.log 2>&1; echo prof=$?
for sm in "96 48" "96 24 24"; do
  python tools/hetero_bench.py --sm $sm --reps 3 > "gpurun_out/r2s11_hetero_f64_$(echo $sm | tr ' ' '_').txt" 2>&1; echo het=$?
done
python tools/hetero_bench.py --sm 96 48 --dtype f32 --n 16384 --reps 3 > gpurun_out/r2s11_hetero_f32_96_48.txt 2>&1; echo het=$?
