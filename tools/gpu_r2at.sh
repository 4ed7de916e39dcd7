O=gpurun_out/r2at; mkdir -p $O
{ for v in default re2; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"
    timeout 300 python tools/quick_bench.py --cfg 3 --pairs 1048576 --reps 3 2>&1 | grep "ms\|hits="
    timeout 300 python tools/quick_bench.py --cfg 6 --pairs 0 --reps 3 2>&1 | grep "ms"
    timeout 600 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "ms"
  done
} > $O/ab.log 2>&1
cat $O/ab.log
