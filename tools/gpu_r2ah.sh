O=gpurun_out/r2ah; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_smem.py -x -q > $O/smemtests.log 2>&1; tail -2 $O/smemtests.log
{ timeout 300 python tools/quick_bench.py --cfg 7 --pairs 0 --reps 3 2>&1 | grep "ms"
  timeout 900 python tools/quick_bench.py --cfg 8 --pairs 0 --reps 1 2>&1 | grep "ms"
  timeout 300 python tools/quick_bench.py --cfg 1 --pairs 1048576 --pair-bits 512 --reps 5 2>&1 | grep "pairs m="
} > $O/ab.log 2>&1
cat $O/ab.log
