set -x
D=gpurun_out/${NS_DIR:-ncu_spadd}
mkdir -p $D
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spadd_tile -c 2 -f -o /tmp/sa python tools/run_op.py spadd C3 > $D/ncu.log 2>&1
ncu -i /tmp/sa.ncu-rep --page raw --csv > $D/raw.csv 2>/dev/null
ncu -i /tmp/sa.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null > /tmp/sa_src.csv
python tools/ncu_lines.py 60 < /tmp/sa_src.csv > $D/lines_both.txt
gzip -c /tmp/sa_src.csv > $D/src.csv.gz
