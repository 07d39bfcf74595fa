D=gpurun_out/addipt; mkdir -p $D
python tools/spadd_fused_time.py C3 C2 > $D/t.txt 2>&1
for ipt in 10 18 22; do
MSP_BUILD_DIR=/tmp/b$ipt MSP_LIB_OUT=/tmp/lib$ipt.so MSP_NVCC_EXTRA="-DMSP_ADD_IPT=$ipt" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$ipt.log 2>&1
MSP_NVCC_EXTRA="-DMSP_ADD_IPT=$ipt" MSP_LIB=/tmp/lib$ipt.so python tools/spadd_fused_time.py C3 C2 >> $D/t.txt 2>&1
done
