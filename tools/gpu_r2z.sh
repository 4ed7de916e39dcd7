O=gpurun_out/r2z; mkdir -p $O
{ echo "== default (swap on resume)"
  for c in 3 6; do timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep "ms"; done
  timeout 300 python tools/quick_bench.py --cfg 1 --pairs 1048576 --reps 5 2>&1 | grep "pairs m="
  timeout 600 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "ms"
  for v in default hy_mix2; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v cfg7/cfg8"
    timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 2>&1 | grep "ms"
    timeout 900 python tools/quick_bench.py --cfg 8 --pairs 0 --reps 1 2>&1 | grep "ms"
  done
} > $O/ab.log 2>&1
cat $O/ab.log
