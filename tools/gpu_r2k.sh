O=gpurun_out/r2k; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_smem.py -x -q > $O/smemtests.log 2>&1; tail -3 $O/smemtests.log
timeout 300 python tools/quick_bench.py --cfg 7 --pairs 65536 --pair-bits 4096 --reps 3 > $O/qb7.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:allpairs_smem -c 1 -o $O/smem_src python tools/prof_allpairs.py 512 4096 1 > $O/ncu.log 2>&1
ncu -i $O/smem_src.ncu-rep --page source --csv --print-source sass > $O/smem_src.csv 2>/dev/null
ncu -i $O/smem_src.ncu-rep --page raw --csv > $O/smem_raw.csv 2>/dev/null
