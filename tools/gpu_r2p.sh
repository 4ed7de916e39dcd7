O=gpurun_out/r2p; mkdir -p $O
for v in default hy8 hy10m; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg7"; timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 2>&1 | grep "all-pairs\|hits"
done > $O/ab.log 2>&1
