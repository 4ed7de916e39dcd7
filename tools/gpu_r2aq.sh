O=gpurun_out/r2aq; mkdir -p $O
{ for v in default xmix2 xg4; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"; timeout 300 python tools/quick_bench.py --cfg 1 --pairs 1048576 --reps 5 2>&1 | grep "pairs m="
  done
} > $O/ab.log 2>&1
cat $O/ab.log
