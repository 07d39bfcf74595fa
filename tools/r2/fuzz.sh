D=gpurun_out/fuzz; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spgemm_fuzz.py -q -rA > $D/tests.log 2>&1; echo t $?
MSP_SPGEMM_ROWACC=0 timeout 900 python -m pytest tests/test_gpu_spgemm_fuzz.py -q > $D/tests_esc.log 2>&1; echo t $?
