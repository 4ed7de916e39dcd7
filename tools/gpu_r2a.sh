set -x
O=gpurun_out/r2a; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt
build/limbmix2 > $O/limbmix2.json 2>&1
timeout 600 python tools/quick_bench.py --cfg 3 --pairs 0 --reps 3 > $O/qb_cfg3.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:allpairs_kernel -c 1 -o $O/ap32_src python tools/prof_allpairs.py 8192 1024 1 > $O/ncu.log 2>&1
ls -la $O
