set -x
for c in C3 C2; do
python tools/exp/spadd_time.py $c >> gpurun_out/spadd_ipt.log 2>&1
MSP_LIB=tools/exp/libmsp_ipt12.so python tools/exp/spadd_time.py $c >> gpurun_out/spadd_ipt.log 2>&1
MSP_LIB=tools/exp/libmsp_ipt16.so python tools/exp/spadd_time.py $c >> gpurun_out/spadd_ipt.log 2>&1
done
