set -x
D=gpurun_out/l1b
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
python tools/spmv_tune.py C3 "CFG=4" "CFG=6" "CFG=7" "CFG=0" >> $D/tune.txt 2>&1
TUNE_DTYPE=float64 python tools/spmv_tune.py C3 "CFG=4" "CFG=6" "CFG=7" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "CFG=4" "CFG=6" "CFG=7" "CFG=0" >> $D/tune.txt 2>&1
TUNE_DTYPE=float32 python tools/spmv_tune.py C4 "CFG=4" "CFG=6" "CFG=7" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C5 "CFG=0" "CFG=4" "CFG=7" >> $D/tune.txt 2>&1
TUNE_DTYPE=float32 python tools/spmv_tune.py C5 "CFG=0" "CFG=4" "CFG=6" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C1 "CFG=4" "CFG=6" "CFG=7" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C2 "VERBOSE=1" "WT_L1=1" >> $D/tune.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_spmv.py tests/test_gpu_spmv_nnz.py -q > $D/tests.log 2>&1; echo tests $?
