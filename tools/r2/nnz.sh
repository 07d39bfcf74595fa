set -x
D=gpurun_out/${NZ_DIR:-nnz1}
mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spmv_nnz.py -x -q > $D/tests.log 2>&1; echo tests $?
MSP_SPMV_WT=2 timeout 900 python -m pytest tests/test_gpu_spmv.py -q > $D/wt2_tests.log 2>&1; echo wt2 $?
