set -x
D=gpurun_out/rowacc
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1; echo build $?
timeout 1200 python -m pytest tests/test_gpu_spgemm_rowacc.py tests/test_gpu_spgemm.py tests/test_abi.py -q -x > $D/tests.log 2>&1; echo tests $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "spgemm" > $D/tests_full.log 2>&1; echo full $?
timeout 900 python tools/spgemm_compare.py C1 C2 C4 > $D/compare.txt 2>&1; echo cmp $?
MSP_SPGEMM_ROWACC=0 timeout 900 python tools/spgemm_compare.py C1 C2 > $D/compare_esc.txt 2>&1; echo cmp0 $?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C2.csv python tools/run_op.py spgemm C2 > $D/ncu.log 2>&1; echo ncu $?
timeout 1200 compute-sanitizer --tool memcheck --print-limit 50 python tools/sanitize_cases.py > $D/memcheck.txt 2>&1; echo memcheck $?
timeout 1200 compute-sanitizer --tool racecheck --print-limit 50 python tools/sanitize_cases.py > $D/racecheck.txt 2>&1; echo racecheck $?
