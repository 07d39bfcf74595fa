set -x
D=gpurun_out/stages; mkdir -p $D
python tools/spmv_tune.py C3 "CFG=9" "CFG=10" "CFG=11" "CFG=4" > $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "CFG=4" "CFG=8" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C5 "CFG=0" >> $D/tune.txt 2>&1
MSP_BUILD_DIR=/tmp/bspin MSP_LIB_OUT=/tmp/libspin.so MSP_NVCC_EXTRA="-DMSP_SPMV_PROD_SPIN=1" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
echo "== spin producer" >> $D/tune.txt
MSP_LIB=/tmp/libspin.so python tools/spmv_tune.py C3 "CFG=9" "CFG=10" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libspin.so python tools/spmv_tune.py C4 "CFG=4" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libspin.so python tools/spmv_tune.py C5 "CFG=0" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libspin.so python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
