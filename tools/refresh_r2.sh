# Re-measure every committed round-2 profile on the current build (one B200):
#   bash tools/refresh_r2.sh [OUTDIR]   -> OUTDIR/r2_*.json|csv|txt (copied to profiles/ by hand)
O=${1:-gpurun_out/r2final}; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/smi.txt 2>&1
git_head=$(cat .git_head 2>/dev/null || echo unknown); echo "$git_head" > $O/build.txt
for w in cfg3 cfg1 cfg2 cfg4 cfg5 cfg6 cfg7 cfg8; do
  case $w in cfg5|cfg8) extra="--steps 5 --warmup 3 --e2e-steps 1";; *) extra="";; esac
  timeout 1200 python bench.py --workload $w $extra > $O/bench_$w.log 2>&1; tail -1 $O/bench_$w.log > $O/r2_bench_$w.json
  echo "$w: $(cut -c1-160 $O/r2_bench_$w.json)"
done
timeout 900 python bench.py --algo C --steps 3 > $O/algoC.log 2>&1; tail -1 $O/algoC.log > $O/r2_bench_cfg3_algoC.json
timeout 900 python bench.py --algo D --steps 3 > $O/algoD.log 2>&1; tail -1 $O/algoD.log > $O/r2_bench_cfg3_algoD.json
timeout 900 python bench.py --impl reference > $O/ref.log 2>&1; tail -1 $O/ref.log > $O/r2_bench_reference_arm.json
echo "algo/ref: $(cut -c1-120 $O/r2_bench_cfg3_algoC.json) | $(cut -c1-120 $O/r2_bench_reference_arm.json)"
# launch list of the default bench command (per-launch times are cold-cache and serialised under ncu)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/r2_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_launch.log 2>&1; echo ncu_launch_rc=$?
# one ncu --set full capture of the hot kernel per workload (roofline.traffic, stall mix)
timeout 1800 python tools/ncu_traffic.py $O cfg3 cfg2 cfg4 cfg6 cfg7 > $O/traffic.log 2>&1; tail -5 $O/traffic.log
ncu -i $O/r2_cfg3.ncu-rep --page source --csv --print-source sass > $O/cfg3_src.csv 2>/dev/null
ncu -i $O/r2_cfg3.ncu-rep --page raw --csv > $O/cfg3_raw.csv 2>/dev/null
python tools/ncu_opmix.py $O/cfg3_src.csv > $O/r2_cfg3_opmix.txt 2>&1
# the reports themselves stay on the box (gpurun copies back at most 64 MiB)
mkdir -p /tmp/ncu_reps && mv $O/*.ncu-rep /tmp/ncu_reps/ 2>/dev/null; gzip -f $O/cfg3_src.csv
# compute-sanitizer is closed on this pool (profiles/r2_compute_sanitizer.txt): the same workload runs
# plainly, checked against construction truth and math.gcd by its own asserts
timeout 900 python tools/sanitize_run.py > $O/r2_sanitize_workload.txt 2>&1; echo "sanitize_run rc=$?" >> $O/r2_sanitize_workload.txt
# microbenchmarks of the limb forms and pipes
mkdir -p build
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/pipemix2 tools/pipemix2.cu && build/pipemix2 > $O/r2_pipemix2.json
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/limbmix2 tools/limbmix2.cu && build/limbmix2 > $O/r2_limbmix2.json
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/limbmix3 tools/limbmix3.cu && build/limbmix3 > $O/r2_limbmix3.json
ls $O
