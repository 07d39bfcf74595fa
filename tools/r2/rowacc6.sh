set -x
D=gpurun_out/rowacc6
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1; echo build $?
timeout 1200 python -m pytest tests/test_gpu_spgemm_rowacc.py tests/test_gpu_spgemm.py tests/test_abi.py -q -x > $D/tests.log 2>&1; echo tests $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "spgemm" > $D/tests_full.log 2>&1; echo full $?
timeout 900 python tools/spgemm_compare.py C1 C2 > $D/compare.txt 2>&1; echo cmp $?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C2.csv python tools/run_op.py spgemm C2 > $D/ncu.log 2>&1; echo ncu $?
for k in wr_symbolic wr_numeric; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -c 1 -f -o /tmp/$k python tools/run_op.py spgemm C2 > $D/ncu_$k.log 2>&1
ncu -i /tmp/$k.ncu-rep --page raw --csv > $D/${k}_raw.csv 2>/dev/null
ncu -i /tmp/$k.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 40 > $D/${k}_lines.txt
done
