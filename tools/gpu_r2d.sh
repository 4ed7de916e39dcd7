O=gpurun_out/r2d; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
for rep in 1 2; do
for v in default t64w18 t32w19 m104 m112 cmpl32; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg3"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 0 --reps 3 2>&1 | grep "all-pairs"
done; done > $O/ab.log 2>&1
unset BULKGCD_SO
