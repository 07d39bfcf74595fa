D=gpurun_out/persist; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spadd.py -q -x > $D/tests.log 2>&1; echo t $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "c3_spadd" >> $D/tests.log 2>&1; echo t $?
python tools/spadd_fused_time.py C3 C2 C1 > $D/t.txt 2>&1
MSP_BUILD_DIR=/tmp/bp0 MSP_LIB_OUT=/tmp/libp0.so MSP_NVCC_EXTRA="-DMSP_ADD_PERSIST=0" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
MSP_NVCC_EXTRA="non-persistent" MSP_LIB=/tmp/libp0.so python tools/spadd_fused_time.py C3 C2 C1 >> $D/t.txt 2>&1
python tools/spadd_fused_time.py C3 C2 >> $D/t.txt 2>&1
