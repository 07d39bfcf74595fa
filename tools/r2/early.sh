set -x
D=gpurun_out/early
mkdir -p $D
python tools/spmv_tune.py C3 "CFG=4" "CFG=8" "CFG=6" "CFG=9" > $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "CFG=4" "CFG=8" "CFG=6" "CFG=9" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C5 "CFG=0" "CFG=4" "CFG=8" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C1 "CFG=4" "CFG=8" >> $D/tune.txt 2>&1
TUNE_DTYPE=float64 python tools/spmv_tune.py C3 "CFG=4" "CFG=8" >> $D/tune.txt 2>&1
