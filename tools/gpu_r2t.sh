O=gpurun_out/r2t; mkdir -p $O
bash tools/ab_cfg3.sh wide mix2 mix4 > $O/ab.log 2>&1
cat $O/ab.log
