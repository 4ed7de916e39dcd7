O=gpurun_out/r2h; mkdir -p $O
for v in default c32w20 c32m104 c32m112 sm104; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg3"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 0 --reps 3 2>&1 | grep "all-pairs"
done > $O/ab.log 2>&1
unset BULKGCD_SO
timeout 600 ncu --set full --import-source on --clock-control none -k regex:pairs_kernel -c 1 -o $O/pairs_exact_src python tools/prof_pairs.py 1048576 0 > $O/ncu.log 2>&1
ncu -i $O/pairs_exact_src.ncu-rep --page source --csv --print-source sass > $O/pairs_exact_src.csv 2>/dev/null
ncu -i $O/pairs_exact_src.ncu-rep --page raw --csv > $O/pairs_exact_raw.csv 2>/dev/null
