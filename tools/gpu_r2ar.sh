O=gpurun_out/r2ar; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_smem.py -x -q > $O/t.log 2>&1; tail -2 $O/t.log
{ timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 2>&1 | grep "ms\|hits="
  timeout 900 python tools/quick_bench.py --cfg 8 --pairs 0 --reps 1 2>&1 | grep "ms\|hits="
} > $O/ab.log 2>&1
cat $O/ab.log
