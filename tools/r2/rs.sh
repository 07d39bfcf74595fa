D=gpurun_out/rs; mkdir -p $D
python tools/spmv_tune.py C3 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" "CFG=15" > $D/tune.txt 2>&1
