O=gpurun_out/r2x; mkdir -p $O
for c in 3 6; do timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep "ms"; done > $O/ab.log 2>&1
cat $O/ab.log
