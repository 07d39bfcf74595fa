D=gpurun_out/wt4; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spmv.py -q -x > $D/tests.log 2>&1; echo t $?
for i in 1 2 3; do python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1; done
python tools/spmv_tune.py C2 "VERBOSE=1" "K=23" "K=31" >> $D/tune.txt 2>&1
TUNE_DTYPE=float32 python tools/spmv_tune.py C2 "VERBOSE=1" >> $D/tune.txt 2>&1
