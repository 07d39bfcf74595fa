set -x
D=gpurun_out/ncu_ws; mkdir -p $D
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_small -s 1 -c 1 -f -o /tmp/ws python tools/run_op.py spgemm C5 > $D/ncu.log 2>&1; echo ncu $?
ncu -i /tmp/ws.ncu-rep --page details --csv > $D/details.csv 2>/dev/null
ncu -i /tmp/ws.ncu-rep --page raw --csv > $D/raw.csv 2>/dev/null
ncu -i /tmp/ws.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 60 > $D/lines.txt
