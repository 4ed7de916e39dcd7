O=gpurun_out/r2r; mkdir -p $O
for v in default p32 p32w24 p32w16; do
  if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
  echo "== $v"; timeout 300 python tools/quick_bench.py --cfg 1 --pairs 1048576 --reps 3 2>&1 | grep "pairs m="
done > $O/ab.log 2>&1
unset BULKGCD_SO

