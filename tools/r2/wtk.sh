D=gpurun_out/wtk; mkdir -p $D
python tools/spmv_tune.py C3 "CFG=-1,WT=2,K=15" "CFG=-1,WT=2,K=11" "CFG=-1,WT=2,K=7" "CFG=-1,WT=2,K=19" > $D/tune.txt 2>&1
python tools/spmv_tune.py C4 "CFG=-1,WT=2,K=7" "CFG=-1,WT=2,K=11" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C5 "CFG=-1,WT=2,K=7" "CFG=-1,WT=2,K=11" >> $D/tune.txt 2>&1
python tools/spmv_tune.py C1 "CFG=-1,WT=2,K=7" >> $D/tune.txt 2>&1
