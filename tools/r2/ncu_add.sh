set -x
D=gpurun_out/ncu_add
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spadd_tile_kernel -c 1 -f -o /tmp/add_C3 python tools/run_op.py spadd_fused C3 > $D/ncu_full.log 2>&1
ncu -i /tmp/add_C3.ncu-rep --page raw --csv > $D/add_C3_raw.csv 2>/dev/null
ncu -i /tmp/add_C3.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 60 > $D/add_C3_lines.txt
ncu -i /tmp/add_C3.ncu-rep --page details --csv > $D/add_C3_details.csv 2>/dev/null
