D=gpurun_out/lb; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spadd.py -q -x > $D/tests.log 2>&1; echo t $?
python tools/spadd_fused_time.py C3 C2 > $D/t.txt 2>&1
MSP_BUILD_DIR=/tmp/blb MSP_LIB_OUT=/tmp/liblb.so MSP_NVCC_EXTRA="-DMSP_LB_BACKOFF=0" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
MSP_NVCC_EXTRA="spin" MSP_LIB=/tmp/liblb.so python tools/spadd_fused_time.py C3 C2 >> $D/t.txt 2>&1
python tools/spadd_fused_time.py C3 C2 >> $D/t.txt 2>&1
