D=gpurun_out/c5s; mkdir -p $D
python tools/spmv_tune.py C5 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" > $D/tune.txt 2>&1
