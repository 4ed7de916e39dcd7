O=gpurun_out/r2e; mkdir -p $O
timeout 600 python bench.py --workload cfg3 > $O/bench_cfg3.log 2>&1
timeout 600 python bench.py --workload cfg2 > $O/bench_cfg2.log 2>&1
for v in default t32w19 t32w20 t32w21; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg3"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 0 --reps 3 2>&1 | grep "all-pairs"
done > $O/ab.log 2>&1
for v in default t32w20; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg4"; timeout 300 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "all-pairs"
done >> $O/ab.log 2>&1
