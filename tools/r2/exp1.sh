set -x
mkdir -p gpurun_out/exp1
python tools/spmv_tune.py C2 "PF=0" "PF=1" "PF=1,NW=4" "PF=0" "PF=1" > gpurun_out/exp1/tune_c2.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/exp1/gputests.log 2>&1; echo tests $?
