D=gpurun_out/addwt; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spadd.py -q -x > $D/tests.log 2>&1; echo t $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "c3_spadd" >> $D/tests.log 2>&1; echo t $?
python tools/spadd_fused_time.py C3 C2 C1 > $D/t.txt 2>&1
MSP_SPADD_WT=0 python tools/spadd_fused_time.py C3 C2 C1 >> $D/t.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C3.csv python tools/run_op.py spadd_fused C3 > $D/ncu.log 2>&1
