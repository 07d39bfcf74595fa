set -x
D=gpurun_out/shapes
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b0.log 2>&1
MSP_NVCC_EXTRA="-DMSP_SPMV_GATHER=1" MSP_BUILD_DIR=/tmp/bg1 MSP_LIB_OUT=/tmp/libg1.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b1.log 2>&1
for c in C1 C3 C4 C5; do
python tools/spmv_tune.py $c "CFG=0" "CFG=4" "CFG=5" "CFG=6" "CFG=7" "CFG=8" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libg1.so python tools/spmv_tune.py $c "CFG=0" "CFG=4" "CFG=6" >> $D/tune_cg.txt 2>&1
done
