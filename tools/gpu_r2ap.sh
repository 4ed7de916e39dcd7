O=gpurun_out/r2ap; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputests.log 2>&1; tail -2 $O/gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 900 python bench.py --workload cfg2 > $O/bench_cfg2.log 2>&1; tail -1 $O/bench_cfg2.log > $O/r2_bench_cfg2.json; cut -c1-200 $O/r2_bench_cfg2.json
timeout 900 python bench.py > $O/bench_cfg3.log 2>&1; tail -1 $O/bench_cfg3.log > $O/r2_bench_cfg3.json; cut -c1-200 $O/r2_bench_cfg3.json
cp profiles/r2_ncu_traffic.json $O/
