set -x
D=gpurun_out/shapes2
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b0.log 2>&1
TUNE_DTYPE=float64 python tools/spmv_tune.py C3 "CFG=0" "CFG=4" "CFG=5" "CFG=6" "CFG=8" >> $D/tune.txt 2>&1
TUNE_DTYPE=float32 python tools/spmv_tune.py C4 "CFG=0" "CFG=4" "CFG=5" "CFG=6" "CFG=8" >> $D/tune.txt 2>&1
TUNE_DTYPE=float32 python tools/spmv_tune.py C5 "CFG=0" "CFG=4" "CFG=6" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C2 "WT=1" "CFG=0" "CFG=6" >> $D/tune.txt 2>&1
bash tools/r2/gprobe.sh
