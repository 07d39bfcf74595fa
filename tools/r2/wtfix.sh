set -x
D=gpurun_out/wtfix
mkdir -p $D
MSP_NVCC_EXTRA="-DMSP_WT_NO_VV_FENCE" MSP_BUILD_DIR=/tmp/bnf MSP_LIB_OUT=/tmp/libnf.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 timeout 900 python -m pytest tests/test_gpu_spmv.py -q -k "c4_full or deterministic or c3_scaled" > $D/fence.log 2>&1; echo fence $?
MSP_LIB=/tmp/libnf.so MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 timeout 900 python -m pytest tests/test_gpu_spmv.py -q -k "c4_full or deterministic or c3_scaled" > $D/nofence.log 2>&1; echo nofence $?
timeout 900 python -m pytest tests/test_gpu_spmv.py tests/test_gpu_dist.py -q > $D/default.log 2>&1; echo default $?
python tools/spmv_tune.py C2 "CFG=-3" > $D/tune.txt 2>&1
