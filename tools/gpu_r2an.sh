O=gpurun_out/r2an; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "all_pairs or band" > $O/t.log 2>&1; tail -2 $O/t.log
{ for v in default c32_0 c32_4 c32_12; do
    if [ $v = default ]; then unset BULKGCD_SO; else export BULKGCD_SO=build/variants/libbulkgcd_$v.so; fi
    echo "== $v"
    for c in 3 6; do timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep "ms\|hits="; done
  done
} > $O/ab.log 2>&1
cat $O/ab.log
