set -x
D=gpurun_out/small
mkdir -p $D
timeout 1500 python -m pytest tests/test_gpu_spgemm_small.py tests/test_gpu_spgemm_rowacc.py tests/test_gpu_spgemm.py tests/test_abi.py -q -x > $D/tests.log 2>&1; echo tests $?
timeout 600 python tools/spgemm_phases.py C1 C2 C4 C5 > $D/phases.txt 2>&1; echo ph $?
MSP_SPGEMM_SMALL=0 timeout 900 python tools/spgemm_phases.py C4 C5 > $D/phases_off.txt 2>&1; echo ph0 $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "spgemm" > $D/tests_full.log 2>&1; echo full $?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C5.csv python tools/run_op.py spgemm C5 > $D/ncu.log 2>&1; echo ncu $?
