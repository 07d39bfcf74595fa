set -x
D=gpurun_out/gath
mkdir -p $D
MSP_NVCC_EXTRA="-DMSP_SPMV_GATHER=1" MSP_BUILD_DIR=/tmp/bg1 MSP_LIB_OUT=/tmp/libg1.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b1.log 2>&1 &
MSP_NVCC_EXTRA="-DMSP_SPMV_GATHER=2" MSP_BUILD_DIR=/tmp/bg2 MSP_LIB_OUT=/tmp/libg2.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b2.log 2>&1 &
wait
for c in C3 C4 C5; do
python tools/spmv_tune.py $c "CFG=0" "CFG=1" "CFG=3" "CFG=4" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libg1.so python tools/spmv_tune.py $c "CFG=0" >> $D/tune_cg.txt 2>&1
MSP_LIB=/tmp/libg2.so python tools/spmv_tune.py $c "CFG=0" >> $D/tune_cs.txt 2>&1
done
