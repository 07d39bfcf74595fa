set -x
D=gpurun_out/ncu_wr
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1
for k in wr_symbolic wr_numeric; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -c 1 -f -o /tmp/$k python tools/run_op.py spgemm C2 > $D/ncu_$k.log 2>&1
ncu -i /tmp/$k.ncu-rep --page raw --csv > $D/${k}_raw.csv 2>/dev/null
ncu -i /tmp/$k.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 40 > $D/${k}_lines.txt
done
