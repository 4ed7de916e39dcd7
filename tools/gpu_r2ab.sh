O=gpurun_out/r2ab; mkdir -p $O
{ for v in g8 g16 g6; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"
    for c in 3 6; do timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep "ms"; done
  done
} > $O/ab.log 2>&1
cat $O/ab.log
