for i in 1 2; do
python tools/spmv_tune.py C2 "CFG=-3" >> gpurun_out/tune_pf2.log 2>&1
MSP_LIB=tools/exp/libmsp_nopf.so python tools/spmv_tune.py C2 "CFG=-3,MSP_LIB=tools/exp/libmsp_nopf.so" >> gpurun_out/tune_pf2.log 2>&1
done
