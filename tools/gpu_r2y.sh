O=gpurun_out/r2y; mkdir -p $O
{ echo "== default (approx hoisted)"
  for c in 3 6; do timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep "ms"; done
  timeout 300 python tools/quick_bench.py --cfg 1 --pairs 1048576 --reps 5 2>&1 | grep "pairs m="
  timeout 600 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "ms"
  for v in w64mix2 cw cm2; do
    echo "== $v cfg4"; BULKGCD_SO=build/variants/libbulkgcd_$v.so timeout 600 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "ms"
  done
} > $O/ab.log 2>&1
cat $O/ab.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
