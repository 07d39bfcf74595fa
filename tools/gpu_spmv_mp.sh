set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k spmv > gpurun_out/gputests_spmv.log 2>&1; echo tests $?
for c in C2 C3 C4; do timeout 900 python tools/spmv_tune.py $c "CFG=-3" "CFG=-3" >> gpurun_out/tune_pf3.log 2>&1; done
