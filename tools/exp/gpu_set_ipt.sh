set -x
python tools/setops_bench.py > gpurun_out/set_ipt12.log 2>&1
MSP_LIB=tools/exp/libmsp_set6.so python tools/setops_bench.py > gpurun_out/set_ipt6.log 2>&1
MSP_LIB=tools/exp/libmsp_set20.so python tools/setops_bench.py > gpurun_out/set_ipt20.log 2>&1
