O=gpurun_out/r2ao; mkdir -p $O
{ for v in default s3c17 s4c17; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"; timeout 300 python tools/e2e_pairs.py 2>&1 | tail -1
  done
  for v in default w64win5; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v cfg4"; timeout 600 python tools/quick_bench.py --cfg 4 --pairs 262144 --pair-bits 2048 --reps 2 2>&1 | grep "ms\|hits="
  done
} > $O/ab.log 2>&1
cat $O/ab.log
