set -x
D=gpurun_out/${TRACE_DIR:-trace5}
mkdir -p $D
timeout 600 python -m pytest tests/test_gpu_spmv.py -x -q > $D/tests.log 2>&1; echo tests $?
python tools/spmv_tune.py C2 "CFG=-3" "CFG=-3" "NW=4" > $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "CFG=-3" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C3 "CFG=-3" >> $D/tune.txt 2>&1
MSP_NVCC_EXTRA=-DMSP_SPMV_TRACE python paper_conf_ipps_daltonbmog15_b200/_build.py --force > $D/build.log 2>&1
python tools/spmv_trace.py C2 > $D/c2.txt 2>&1
