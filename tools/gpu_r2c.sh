O=gpurun_out/r2c; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
for rep in 1 2; do
for v in cmpl split; do
  if [ $v = cmpl ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_split.so; fi
  for c in 3 4 6; do echo "== $v cfg$c"; timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep -v "^lib\|generated"; done
done; done > $O/ab.log 2>&1
unset BULKGCD_SO
