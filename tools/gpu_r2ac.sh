O=gpurun_out/r2ac; mkdir -p $O
{ for v in default rsag4; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"
    timeout 300 python tools/quick_bench.py --cfg 3 --pairs 1048576 --reps 5 2>&1 | grep "ms"
  done
} > $O/ab.log 2>&1
cat $O/ab.log
