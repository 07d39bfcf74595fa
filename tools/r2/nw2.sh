D=gpurun_out/nw2; mkdir -p $D
for cfg in "5 2 4" "5 2 5" "5 3 3" "4 3 3"; do
set -- $cfg
MSP_BUILD_DIR=/tmp/bm$1$2$3 MSP_LIB_OUT=/tmp/libm$1$2$3.so MSP_NVCC_EXTRA="-DMSP_WT_NW=$1 -DMSP_WT_STAGES=$2 -DMSP_WT_NSUB=$3" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$1$2$3.log 2>&1
echo "== nw $1 stages $2 nsub $3" >> $D/tune.txt
MSP_LIB=/tmp/libm$1$2$3.so python tools/spmv_tune.py C2 "VERBOSE=1" "K=27" >> $D/tune.txt 2>&1
done
