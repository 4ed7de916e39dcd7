O=gpurun_out/r2aa; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
{ for v in default noswap; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"
    timeout 600 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "ms\|Error\|error"
  done
  unset BULKGCD_SO
  echo "== default cfg3/cfg6/cfg7"
  for c in 3 6 7; do timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep "ms"; done
} > $O/ab.log 2>&1
cat $O/ab.log
