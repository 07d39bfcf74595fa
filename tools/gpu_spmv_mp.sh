mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c4gemm.csv python tools/run_op.py spgemm C4 > /dev/null 2>&1
