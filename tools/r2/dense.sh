set -x
D=gpurun_out/dense
mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_spgemm_segmented.py -q > $D/tests.log 2>&1; echo tests $?
python tools/dense_spgemm.py 500 1000 2000 > $D/dense.txt 2>&1
MSP_SPGEMM_SEGMENTED=0 python tools/dense_spgemm.py 500 1000 > $D/dense_esc.txt 2>&1
python tools/spgemm_compare.py C2 C4 > $D/compare.txt 2>&1
