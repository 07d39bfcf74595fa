set -x
D=gpurun_out/ncu_add2; mkdir -p $D
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spadd_tile -c 1 -f -o /tmp/add python tools/run_op.py spadd_fused C3 > $D/ncu.log 2>&1; echo ncu $?
ncu -i /tmp/add.ncu-rep --page details --csv > $D/details.csv 2>/dev/null
ncu -i /tmp/add.ncu-rep --page raw --csv > $D/raw.csv 2>/dev/null
ncu -i /tmp/add.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 60 > $D/lines.txt
