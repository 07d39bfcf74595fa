D=gpurun_out/wtl1; mkdir -p $D
for i in 1 2; do python tools/spmv_tune.py C2 "VERBOSE=1" "WT_L1=1" >> $D/tune.txt 2>&1; done
