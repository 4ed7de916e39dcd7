# ncu of the current build: cfg3 all-pairs and cfg2 exact pairs (full set + source), launch list of bench.py
O=gpurun_out/r2v; mkdir -p $O
timeout 900 python tools/ncu_traffic.py $O cfg3 cfg2 > $O/traffic.log 2>&1; tail -3 $O/traffic.log
for w in cfg3 cfg2; do
  ncu -i $O/r2_$w.ncu-rep --page source --csv --print-source sass > $O/${w}_src.csv 2>/dev/null
  ncu -i $O/r2_$w.ncu-rep --page raw --csv > $O/${w}_raw.csv 2>/dev/null
done
timeout 600 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/plain.log 2>&1; echo plain_rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_launch.log 2>&1; echo ncu_launch_rc=$?
ls -la $O
