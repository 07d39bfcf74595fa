D=gpurun_out/small2; mkdir -p $D
timeout 600 python tools/spgemm_phases.py C4 C5 > $D/phases.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C5.csv python tools/run_op.py spgemm C5 > $D/ncu.log 2>&1
