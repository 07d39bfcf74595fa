set -x
mkdir -p gpurun_out/tl
timeout 600 python -m pytest tests -m gpu -x -q -k "spmv" > gpurun_out/gputests_spmv.log 2>&1; echo tests $?
MSP_SPMV_FLAGS=16 MSP_SPMV_TL_FILE=gpurun_out/tl/mp8.txt MSP_SPMV_CFG=-2 python tools/run_op.py spmv C2 5
timeout 900 python tools/spmv_tune.py C2 "CFG=-1" "CFG=-2" "CFG=-2,PF=3" "CFG=-2,PF=4" "CFG=-2,ST=3,K=21" "CFG=-2,K=15,MB=2" "CFG=-2,NW=16,K=15" > gpurun_out/tune_mp11.log 2>&1
timeout 900 python tools/spmv_tune.py C3 "CFG=-2" "CFG=-2,NW=4,K=15" >> gpurun_out/tune_mp11.log 2>&1
timeout 900 python tools/spmv_tune.py C4 "CFG=-2" "CFG=-2,K=15,MB=2" >> gpurun_out/tune_mp11.log 2>&1
