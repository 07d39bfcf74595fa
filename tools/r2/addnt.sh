D=gpurun_out/addnt2; mkdir -p $D
python tools/spadd_fused_time.py C3 C2 > $D/t.txt 2>&1
for cfg in "128 14" "128 12" "128 16" "64 14" "64 20" "96 14"; do
set -- $cfg
MSP_BUILD_DIR=/tmp/ba$1$2 MSP_LIB_OUT=/tmp/liba$1$2.so MSP_NVCC_EXTRA="-DMSP_ADD_NT=$1 -DMSP_ADD_IPT=$2" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$1$2.log 2>&1
MSP_NVCC_EXTRA="NT=$1 IPT=$2" MSP_LIB=/tmp/liba$1$2.so python tools/spadd_fused_time.py C3 C2 >> $D/t.txt 2>&1
done
