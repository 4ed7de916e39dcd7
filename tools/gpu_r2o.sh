O=gpurun_out/r2o; mkdir -p $O
timeout 600 ncu --set full --import-source on --clock-control none -k regex:allpairs_hybrid -c 1 -o $O/hy_src python tools/prof_allpairs.py 512 4096 1 > $O/ncu.log 2>&1
ncu -i $O/hy_src.ncu-rep --page source --csv --print-source sass > $O/hy_src.csv 2>/dev/null
ncu -i $O/hy_src.ncu-rep --page raw --csv > $O/hy_raw.csv 2>/dev/null
