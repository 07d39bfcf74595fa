D=gpurun_out/c4; mkdir -p $D
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C4.csv python tools/run_op.py spgemm C4 > $D/ncu.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C3add.csv python tools/run_op.py spadd_fused C3 > $D/ncu2.log 2>&1
