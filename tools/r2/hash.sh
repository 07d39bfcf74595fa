D=gpurun_out/hash; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spgemm_rowacc.py tests/test_gpu_fullsize.py -k "not esc_tile and (rowacc or c2_spgemm)" -q > $D/tests.log 2>&1; echo t $?
timeout 600 python tools/spgemm_phases.py C2 --reps 8 > $D/phases.txt 2>&1
