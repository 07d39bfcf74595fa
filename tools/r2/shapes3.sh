set -x
D=gpurun_out/shapes3
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b0.log 2>&1
MSP_NVCC_EXTRA="-DMSP_SPMV_GATHER=3" MSP_BUILD_DIR=/tmp/bg3 MSP_LIB_OUT=/tmp/libg3.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b3.log 2>&1
timeout 600 python -m pytest tests/test_gpu_spmv.py -q -x > $D/t_default.log 2>&1; echo t0 $?
MSP_SPMV_CFG=6 timeout 600 python -m pytest tests/test_gpu_spmv.py -q -x > $D/t_cfg6.log 2>&1; echo t6 $?
python tools/spmv_tune.py C4 "CFG=0" "CFG=4" "CFG=5" "CFG=6" "CFG=8" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C3 "CFG=0" "CFG=4" "CFG=6" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C5 "CFG=0" "CFG=4" >> $D/tune.txt 2>&1
MSP_LIB=/tmp/libg3.so python tools/spmv_tune.py C5 "CFG=0" "CFG=4" >> $D/tune_g3.txt 2>&1
MSP_LIB=/tmp/libg3.so python tools/spmv_tune.py C3 "CFG=6" >> $D/tune_g3.txt 2>&1
MSP_LIB=/tmp/libg3.so python tools/spmv_tune.py C4 "CFG=0" >> $D/tune_g3.txt 2>&1
