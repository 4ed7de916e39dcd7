O=gpurun_out/r2w; mkdir -p $O
for v in default oe0; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v"; timeout 300 python tools/quick_bench.py --cfg 1 --pairs 1048576 --reps 5 2>&1 | grep "pairs m="
  timeout 300 python tools/quick_bench.py --cfg 1 --pairs 262144 --pair-bits 2048 --reps 5 2>&1 | grep "pairs m="
done > $O/ab.log 2>&1
unset BULKGCD_SO
echo "== default cfg4" >> $O/ab.log; timeout 600 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 3 2>&1 | grep "ms" >> $O/ab.log
cat $O/ab.log
