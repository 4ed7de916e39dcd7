O=gpurun_out/r2as; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputests.log 2>&1; tail -2 $O/gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
for w in cfg7 cfg8; do
  case $w in cfg8) extra="--steps 5 --warmup 3 --e2e-steps 1";; *) extra="";; esac
  timeout 1200 python bench.py --workload $w $extra > $O/bench_$w.log 2>&1; tail -1 $O/bench_$w.log > $O/r2_bench_$w.json
  echo "$w: $(cut -c1-140 $O/r2_bench_$w.json)"
done
cp profiles/r2_ncu_traffic.json $O/r2_ncu_traffic.json
timeout 900 python tools/ncu_traffic.py $O cfg7 > $O/traffic.log 2>&1; tail -1 $O/traffic.log
rm -f $O/*.ncu-rep
