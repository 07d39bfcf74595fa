set -x
D=gpurun_out/wtdbg2
mkdir -p $D
MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 MSP_SPMV_K=7 python tools/wt_debug.py > $D/k7.txt 2>&1
MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 MSP_SPMV_K=27 python tools/wt_debug.py > $D/k27.txt 2>&1
MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 timeout 900 python -m pytest tests/test_gpu_spmv.py -q > $D/wt2_tests.log 2>&1; echo wt2 $?
python tools/spmv_tune.py C2 "CFG=-3" > $D/tune.txt 2>&1
