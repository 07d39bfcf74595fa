D=gpurun_out/acc2; mkdir -p $D
python tools/spmv_tune.py C2 "VERBOSE=1" > $D/tune.txt 2>&1
MSP_BUILD_DIR=/tmp/ba2 MSP_LIB_OUT=/tmp/liba2.so MSP_NVCC_EXTRA="-DMSP_WT_ACC2=1" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
echo "== acc2" >> $D/tune.txt
MSP_LIB=/tmp/liba2.so python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/liba2.so python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
