O=gpurun_out/r2f; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
for c in 3 4 6; do echo "== cfg$c"; timeout 300 python tools/quick_bench.py --cfg $c --pairs 0 --reps 3 2>&1 | grep "all-pairs\|hits"; done > $O/qb.log 2>&1
timeout 600 python bench.py --workload cfg3 > $O/bench_cfg3.log 2>&1
