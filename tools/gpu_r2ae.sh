O=gpurun_out/r2ae; mkdir -p $O
{ for v in g64_4 g64_8; do
    export BULKGCD_SO=build/variants/libbulkgcd_$v.so; echo "== $v"
    timeout 600 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "ms"
  done
  for v in default hyg8; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"; timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 2>&1 | grep "ms"
  done
} > $O/ab.log 2>&1
cat $O/ab.log
