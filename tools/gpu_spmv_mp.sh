set -x
mkdir -p gpurun_out
timeout 900 python tools/spmv_tune.py C2 "CFG=-1" "CFG=-4,K=19" "CFG=-4,K=15" "CFG=-4,K=11" > gpurun_out/tune_pipe.log 2>&1
timeout 900 python tools/spmv_tune.py C3 "CFG=0" "CFG=-4,K=15" "CFG=-4,K=11" "CFG=-4,K=7" >> gpurun_out/tune_pipe.log 2>&1
timeout 900 python tools/spmv_tune.py C4 "CFG=0" "CFG=-4,K=7" "CFG=-4,K=11" >> gpurun_out/tune_pipe.log 2>&1
MSP_SPMV_CFG=-4 timeout 600 python -m pytest tests -m gpu -x -q -k "spmv" > gpurun_out/gputests_pipe.log 2>&1; echo tests $?
