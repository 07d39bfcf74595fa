set -x
D=gpurun_out/fused
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1; echo build $?
timeout 1200 python -m pytest tests/test_gpu_spadd.py tests/test_gpu_setops.py tests/test_abi.py -q -x > $D/tests.log 2>&1; echo tests $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "spadd or set_operation" > $D/tests_full.log 2>&1; echo full $?
timeout 600 python tools/setops_bench.py > $D/setops.txt 2>&1; echo setops $?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/spadd_launches.csv python tools/run_op.py spadd_fused C3 2 > $D/ncu1.log 2>&1; echo ncu $?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/spadd2_launches.csv python tools/run_op.py spadd C3 2 > $D/ncu2.log 2>&1; echo ncu2 $?
timeout 1500 python bench.py > $D/bench.log 2>&1; echo bench $?
