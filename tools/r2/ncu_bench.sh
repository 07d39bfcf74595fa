set -x
D=gpurun_out/${NB_DIR:-nb1}
mkdir -p $D
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_wt -c 1 -f -o /tmp/spmv_C2 python tools/run_op.py spmv C2 > $D/ncu.log 2>&1
ncu -i /tmp/spmv_C2.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 60 > $D/lines.txt
ncu -i /tmp/spmv_C2.ncu-rep --page raw --csv > $D/raw.csv 2>/dev/null
timeout 1200 python bench.py > $D/bench.log 2>&1; echo bench $?
