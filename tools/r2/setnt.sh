D=gpurun_out/setnt; mkdir -p $D
python tools/r2/setq.py default > $D/t.txt 2>&1
for cfg in "128 12" "128 16" "256 16" "512 8"; do
set -- $cfg
MSP_BUILD_DIR=/tmp/bs$1$2 MSP_LIB_OUT=/tmp/libs$1$2.so MSP_NVCC_EXTRA="-DMSP_SET_NT=$1 -DMSP_SET_IPT=$2" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$1$2.log 2>&1
MSP_LIB=/tmp/libs$1$2.so python tools/r2/setq.py "NT=$1 IPT=$2" >> $D/t.txt 2>&1
done
