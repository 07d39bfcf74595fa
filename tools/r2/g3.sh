D=gpurun_out/g3; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spmv.py -q -x > $D/tests.log 2>&1; echo t $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "c3_spmv" >> $D/tests.log 2>&1; echo t $?
python tools/spmv_tune.py C3 "VERBOSE=1" > $D/tune.txt 2>&1
