D=gpurun_out/c1; mkdir -p $D
timeout 1500 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_spgemm_segmented.py tests/test_gpu_spgemm_small.py tests/test_gpu_spgemm_fuzz.py -q -x > $D/tests.log 2>&1; echo t $?
timeout 600 python tools/spgemm_phases.py C1 C2 C4 --reps 10 > $D/phases.txt 2>&1
