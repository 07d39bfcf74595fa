set -x
D=gpurun_out/wtncu; mkdir -p $D
TUNE_DTYPE=float32 python tools/spmv_tune.py C2 "VERBOSE=1" > $D/tune.txt 2>&1
MSP_BUILD_DIR=/tmp/bw3 MSP_LIB_OUT=/tmp/libw3.so MSP_NVCC_EXTRA="-DMSP_WT_STAGES=3" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b3.log 2>&1
echo "== stages 3 (previous default)" >> $D/tune.txt
MSP_LIB=/tmp/libw3.so TUNE_DTYPE=float32 python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libw3.so python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_wt -c 1 -f -o /tmp/wt python tools/run_op.py spmv C2 > $D/ncu.log 2>&1
ncu -i /tmp/wt.ncu-rep --page raw --csv > $D/raw.csv 2>/dev/null
ncu -i /tmp/wt.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 60 > $D/lines.txt
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_bench.csv python bench.py --steps 1 --warmup 3 --spmv-reps 2 --no-e2e --no-cpu --no-table > $D/bench_ncu.log 2>&1
timeout 900 python bench.py --no-table > $D/bench.log 2>&1
