O=gpurun_out/r2n; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_smem.py -x -q > $O/smemtests.log 2>&1; tail -3 $O/smemtests.log
timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 > $O/qb7.log 2>&1
timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 --flags smem >> $O/qb7.log 2>&1
timeout 900 python bench.py --workload cfg8 --steps 2 --warmup 3 --e2e-steps 1 --no-cpu-baseline > $O/bench_cfg8.log 2>&1; tail -1 $O/bench_cfg8.log | cut -c1-300
