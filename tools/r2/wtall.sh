set -x
D=gpurun_out/${WA_DIR:-wtall1}
mkdir -p $D
MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 timeout 900 python -m pytest tests/test_gpu_spmv.py -q > $D/wt2_tests.log 2>&1; echo wt2 $?
MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -k "c3_spmv" > $D/wt2_c3.log 2>&1; echo wt2c3 $?
