D=gpurun_out/lb2; mkdir -p $D
python tools/spadd_fused_time.py C3 C2 > $D/t.txt 2>&1
for cfg in "1 16" "1 64" "1 4"; do
set -- $cfg
MSP_BUILD_DIR=/tmp/bl$1$2 MSP_LIB_OUT=/tmp/libl$1$2.so MSP_NVCC_EXTRA="-DMSP_LB_BACKOFF=$1 -DMSP_LB_SPINS=$2" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$1$2.log 2>&1
MSP_NVCC_EXTRA="backoff spins $2" MSP_LIB=/tmp/libl$1$2.so python tools/spadd_fused_time.py C3 C2 >> $D/t.txt 2>&1
done
python tools/spadd_fused_time.py C3 C2 >> $D/t.txt 2>&1
