set -x
D=gpurun_out/${WT_DIR:-wt4}
mkdir -p $D
timeout 600 python -m pytest tests/test_gpu_spmv.py -x -q > $D/tests.log 2>&1; echo tests $?
python tools/spmv_tune.py C2 "CFG=-3" "CFG=-3" "WT=0" > $D/tune.txt 2>&1
MSP_NVCC_EXTRA=-DMSP_SPMV_TRACE MSP_BUILD_DIR=/tmp/btr MSP_LIB_OUT=/tmp/libtr.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1
MSP_LIB=/tmp/libtr.so python tools/spmv_wt_trace.py C2 > $D/c2.txt 2>&1
