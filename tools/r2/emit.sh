D=gpurun_out/emit; mkdir -p $D
timeout 600 python tools/spgemm_phases.py C2 --reps 5 > $D/phases.txt 2>&1
MSP_BUILD_DIR=/tmp/be MSP_LIB_OUT=/tmp/libe.so MSP_NVCC_EXTRA="-DWR_EMIT_SERIAL=1" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
MSP_LIB=/tmp/libe.so timeout 600 python tools/spgemm_phases.py C2 --reps 5 >> $D/phases.txt 2>&1
MSP_LIB=/tmp/libe.so timeout 900 python -m pytest tests/test_gpu_spgemm_rowacc.py tests/test_gpu_fullsize.py -k "not esc_tile and not small_path and (rowacc or c2_spgemm)" -q > $D/tests.log 2>&1; echo t $?
