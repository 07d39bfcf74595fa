set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "spgemm" > gpurun_out/gputests_spgemm.log 2>&1; echo tests $?
timeout 1200 python tools/sweep.py --configs C2,C4 --ops spgemm --out gpurun_out/sweep_gemm.json > gpurun_out/sweep_gemm.log 2>&1; echo sweep $?
