set -x
D=gpurun_out/sweep
mkdir -p $D
timeout 600 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_spgemm_segmented.py -q > $D/tests.log 2>&1; echo tests $?
python tools/spgemm_compare.py C4 > $D/compare_c4.txt 2>&1
timeout 2400 python tools/predict_sweep.py --json $D/predict.json > $D/predict.txt 2>&1; echo sweep $?
