D=gpurun_out/c5test; mkdir -p $D
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -x -k "c5_spgemm" > $D/tests.log 2>&1; echo t $?
