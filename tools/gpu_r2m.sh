O=gpurun_out/r2m; mkdir -p $O
for rep in 1 2; do for v in default c96w20; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg3"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 0 --reps 3 2>&1 | grep "all-pairs"
  echo "== $v cfg6"; timeout 300 python tools/quick_bench.py --cfg 6 --pairs 0 --reps 3 2>&1 | grep "all-pairs"
done; done > $O/ab.log 2>&1
