D=gpurun_out/shapes4; mkdir -p $D
python tools/spmv_tune.py C3 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" "CFG=15" > $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" "CFG=15" >> $D/tune.txt 2>&1
TUNE_DTYPE=float32 python tools/spmv_tune.py C4 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C1 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" >> $D/tune.txt 2>&1
