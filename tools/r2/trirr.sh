set -x
D=gpurun_out/trirr
mkdir -p $D
MSP_NVCC_EXTRA=-DMSP_SPMV_TRACE MSP_BUILD_DIR=/tmp/btr MSP_LIB_OUT=/tmp/libtr.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1
MSP_LIB=/tmp/libtr.so python tools/spmv_trace.py C3 > $D/c3.txt 2>&1
MSP_LIB=/tmp/libtr.so python tools/spmv_trace.py C4 > $D/c4.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -f -o /tmp/c3 python tools/run_op.py spmv C3 > $D/ncu.log 2>&1
ncu -i /tmp/c3.ncu-rep --page raw --csv > $D/c3_raw.csv 2>/dev/null
ncu -i /tmp/c3.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 50 > $D/c3_lines.txt
