D=gpurun_out/nw; mkdir -p $D
python tools/spmv_tune.py C2 "VERBOSE=1" > $D/tune.txt 2>&1
for cfg in "10 4" "9 4" "7 4" "10 5" "5 4"; do
set -- $cfg
MSP_BUILD_DIR=/tmp/bn$1$2 MSP_LIB_OUT=/tmp/libn$1$2.so MSP_NVCC_EXTRA="-DMSP_WT_NW=$1 -DMSP_WT_STAGES=$2" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$1$2.log 2>&1
echo "== nw $1 stages $2" >> $D/tune.txt
MSP_LIB=/tmp/libn$1$2.so python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
done
