D=gpurun_out/wtwarm; mkdir -p $D
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none --csv --log-file $D/warm_4x4.csv python tools/run_op.py spmv C2 6 > $D/n1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/cold_4x4.csv python tools/run_op.py spmv C2 6 > $D/n2.log 2>&1
MSP_BUILD_DIR=/tmp/bw3 MSP_LIB_OUT=/tmp/libw3.so MSP_NVCC_EXTRA="-DMSP_WT_STAGES=3" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b3.log 2>&1
MSP_LIB=/tmp/libw3.so timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none --csv --log-file $D/warm_3x6.csv python tools/run_op.py spmv C2 6 > $D/n3.log 2>&1
MSP_LIB=/tmp/libw3.so timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/cold_3x6.csv python tools/run_op.py spmv C2 6 > $D/n4.log 2>&1
