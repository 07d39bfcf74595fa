set -x
D=gpurun_out/${SG_DIR:-seg2}
mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spgemm_segmented.py tests/test_gpu_spgemm.py tests/test_gpu_fullsize.py tests/test_gpu_dist.py -q > $D/tests.log 2>&1; echo tests $?
