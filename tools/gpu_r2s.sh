# Round-2 re-entry: GPU tests, cfg3 bench line, launch list and ncu full capture on the current build.
O=gpurun_out/r2s; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $O/gputests.log 2>&1; tail -3 $O/gputests.log
timeout 600 python bench.py > $O/bench_cfg3.log 2>&1; tail -1 $O/bench_cfg3.log > $O/r2_bench_cfg3.json; cut -c1-400 $O/r2_bench_cfg3.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $O/ncu_launch.log 2>&1; echo ncu_launch_rc=$?
timeout 900 python tools/ncu_traffic.py $O cfg3 > $O/traffic.log 2>&1; tail -2 $O/traffic.log
ncu -i $O/r2_cfg3.ncu-rep --page source --csv --print-source sass > $O/cfg3_src.csv 2>/dev/null
ncu -i $O/r2_cfg3.ncu-rep --page raw --csv > $O/cfg3_raw.csv 2>/dev/null
ls -la $O
