O=gpurun_out/r2q; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 > $O/qb7.log 2>&1
timeout 1200 python bench.py --workload cfg8 --steps 3 --warmup 3 --e2e-steps 1 > $O/bench_cfg8.log 2>&1; tail -1 $O/bench_cfg8.log | cut -c1-300
