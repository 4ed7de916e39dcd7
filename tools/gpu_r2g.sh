O=gpurun_out/r2g; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_smem.py -x -q -s -k "beta_positive" > $O/beta.log 2>&1; tail -5 $O/beta.log
timeout 1200 python bench.py --workload cfg8 --steps 2 --warmup 3 --e2e-steps 1 > $O/bench_cfg8.log 2>&1; tail -1 $O/bench_cfg8.log | cut -c1-400
