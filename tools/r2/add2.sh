D=gpurun_out/add2; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spadd.py -q -x > $D/tests.log 2>&1; echo t $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "c3_spadd" >> $D/tests.log 2>&1; echo t $?
python tools/spadd_fused_time.py C3 C2 C1 > $D/t.txt 2>&1
