D=gpurun_out/wtsweep2; mkdir -p $D
python tools/spmv_tune.py C2 "VERBOSE=1" > $D/tune.txt 2>&1
for cfg in "4 4" "4 5" "5 4" "5 3" "6 3" "3 6"; do
set -- $cfg
MSP_BUILD_DIR=/tmp/bw$1$2 MSP_LIB_OUT=/tmp/libw$1$2.so MSP_NVCC_EXTRA="-DMSP_WT_STAGES=$1 -DMSP_WT_NSUB=$2" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$1$2.log 2>&1
echo "== stages $1 nsub $2" >> $D/tune.txt
MSP_LIB=/tmp/libw$1$2.so python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
done
