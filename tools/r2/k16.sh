D=gpurun_out/k16; mkdir -p $D
python tools/spmv_tune.py C3 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" "CFG=15" > $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "VERBOSE=1" "CFG=13" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C5 "VERBOSE=1" "CFG=13" >> $D/tune.txt 2>&1
