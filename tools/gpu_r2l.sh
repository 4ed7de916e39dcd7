O=gpurun_out/r2l; mkdir -p $O
for v in default s104w19 s112w18 c104w19 c112w18 two8; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  [ -f "${BULKGCD_SO:-paper_conf_ipps_fujitani15_b200/libbulkgcd.so}" ] || continue
  echo "== $v cfg3"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 0 --reps 3 2>&1 | grep "all-pairs"
done > $O/ab.log 2>&1
for v in default w64t32 w64t64; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg4"; timeout 300 python tools/quick_bench.py --cfg 4 --pairs 0 --reps 2 2>&1 | grep "all-pairs"
done >> $O/ab.log 2>&1
unset BULKGCD_SO
timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 2>&1 | grep "all-pairs" >> $O/ab.log
