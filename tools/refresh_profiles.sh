# Re-measure every committed bench line on the current build (one B200): tools/refresh_profiles.sh OUTDIR
out=${1:-gpurun_out/refresh}; mkdir -p $out
for w in cfg1 cfg2 cfg3 cfg4 cfg5 cfg6 cfg7; do
  timeout 900 python bench.py --workload $w > $out/bench_$w.log 2>&1; tail -1 $out/bench_$w.log > $out/r1_bench_$w.json
done
timeout 600 python bench.py --algo C > $out/algoC.log 2>&1; tail -1 $out/algoC.log > $out/r1_bench_cfg3_algoC.json
timeout 600 python bench.py --algo D > $out/algoD.log 2>&1; tail -1 $out/algoD.log > $out/r1_bench_cfg3_algoD.json
timeout 600 python bench.py --impl reference > $out/ref.log 2>&1; tail -1 $out/ref.log > $out/r1_bench_reference_arm.json
