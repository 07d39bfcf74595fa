D=gpurun_out/segt; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spgemm_segmented.py -q > $D/tests.log 2>&1; echo t $?
