#!/bin/bash
# Time each build/variants/libbulkgcd_<name>.so on cfg3 (tuning aid): tools/run_variants.sh name1 name2 ...
for v in "$@"; do
  echo "== $v"
  BULKGCD_SO=build/variants/libbulkgcd_$v.so timeout 300 python tools/quick_bench.py --cfg ${CFG:-3} --pairs ${PAIRS:-0} --reps ${REPS:-3} 2>&1 | grep -v "^lib\|generated"
done
