O=gpurun_out/r2ad; mkdir -p $O
timeout 300 python tools/quick_bench.py --cfg 3 --pairs 1048576 --reps 5 2>&1 | grep "ms" > $O/ab.log
timeout 300 python tools/quick_bench.py --cfg 1 --pairs 262144 --pair-bits 2048 --reps 5 2>&1 | grep "pairs m=" >> $O/ab.log
cat $O/ab.log
timeout 1200 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
