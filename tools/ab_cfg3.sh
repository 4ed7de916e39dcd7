# cfg3 all-pairs + 2^20 1024-bit pairs (exact, RSA) for the default build and build/variants/libbulkgcd_<v>.so
for v in default "$@"; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 1048576 --reps 3 2>&1 | grep "ms"
done
