O=gpurun_out/r2u; mkdir -p $O
bash tools/ab_cfg3.sh split mix3 > $O/ab.log 2>&1
for v in default split; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg6"; timeout 300 python tools/quick_bench.py --cfg 6 --pairs 0 --reps 3 2>&1 | grep "ms"
done >> $O/ab.log 2>&1
unset BULKGCD_SO
cat $O/ab.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
