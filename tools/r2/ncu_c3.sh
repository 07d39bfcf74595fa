set -x
D=gpurun_out/ncu_c3; mkdir -p $D
timeout 600 python -m pytest tests/test_gpu_spmv.py -q -x > $D/tests.log 2>&1; echo tests $?
python tools/spmv_tune.py C3 "VERBOSE=1" > $D/tune.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -f -o /tmp/c3 python tools/run_op.py spmv C3 > $D/ncu.log 2>&1; echo ncu $?
ncu -i /tmp/c3.ncu-rep --page details --csv > $D/details.csv 2>/dev/null
ncu -i /tmp/c3.ncu-rep --page raw --csv > $D/raw.csv 2>/dev/null
ncu -i /tmp/c3.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 50 > $D/lines.txt
