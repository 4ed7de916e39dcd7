# A/B of the ONE_ENTRY resume (kernels.cuh euclid_loop): tools/ab_resume.sh [variant names...]
for v in default "$@"; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v cfg3"; timeout 300 python tools/quick_bench.py --cfg 3 --pairs 1048576 --reps 3 2>&1 | grep -v "^lib\|generated"
  echo "== $v cfg4"; timeout 300 python tools/quick_bench.py --cfg 4 --pairs 262144 --pair-bits 2048 --reps 3 2>&1 | grep -v "^lib\|generated"
done
