O=gpurun_out/r2b; mkdir -p $O
build/pipemix2 > $O/pipemix2.json 2>&1
build/limbmix3 > $O/limbmix3.json 2>&1
