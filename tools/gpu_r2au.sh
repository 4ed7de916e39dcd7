O=gpurun_out/r2au; mkdir -p $O
{ for v in default c32w18 w18; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 0 --reps 3 2>&1 | grep "ms\|hits="
  done
} > $O/ab.log 2>&1
cat $O/ab.log
