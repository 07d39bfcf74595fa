set -x
D=gpurun_out/${IR_DIR:-irr1}
mkdir -p $D
for c in C3 C4; do
python tools/spmv_tune.py $c "CFG=-3" "CFG=-1,WT=2,K=7" "CFG=-1,WT=2,K=11" "CFG=-1,WT=2,K=15" "CFG=-1,WT=0,K=7" >> $D/tune.txt 2>&1
done
python tools/spmv_tune.py C5 "CFG=-3" "CFG=-1,WT=2,K=7" >> $D/tune.txt 2>&1
