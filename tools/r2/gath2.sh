D=gpurun_out/gath2; mkdir -p $D
python tools/spmv_tune.py C3 "VERBOSE=1" > $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "VERBOSE=1" >> $D/tune.txt 2>&1
for g in 0 4; do
MSP_BUILD_DIR=/tmp/bg$g MSP_LIB_OUT=/tmp/libg$g.so MSP_NVCC_EXTRA="-DMSP_SPMV_GATHER=$g" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$g.log 2>&1
echo "== gather $g" >> $D/tune.txt
MSP_LIB=/tmp/libg$g.so python tools/spmv_tune.py C3 "VERBOSE=1" "CFG=4" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libg$g.so python tools/spmv_tune.py C4 "VERBOSE=1" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libg$g.so python tools/spmv_tune.py C5 "VERBOSE=1" >> $D/tune.txt 2>&1
done
