set -x
D=gpurun_out/${NCU_DIR:-ncu_spmv}
mkdir -p $D
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -f -o /tmp/spmv_C2 python tools/run_op.py spmv ${CFG:-C2} > $D/ncu.log 2>&1
ncu -i /tmp/spmv_C2.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 80 > $D/lines.txt
ncu -i /tmp/spmv_C2.ncu-rep --page source --csv --print-source sass 2>/dev/null | python tools/ncu_sass_top.py 80 > $D/sass_top.txt
ncu -i /tmp/spmv_C2.ncu-rep --page raw --csv > $D/raw.csv 2>/dev/null
ncu -i /tmp/spmv_C2.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > $D/sass.csv.gz
