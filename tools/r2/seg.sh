D=gpurun_out/seg; mkdir -p $D
timeout 1500 python -m pytest tests/test_gpu_spgemm_segmented.py tests/test_gpu_spgemm_small.py tests/test_gpu_spgemm.py -q -x > $D/tests.log 2>&1; echo tests $?
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "spgemm" > $D/tests_full.log 2>&1; echo full $?
timeout 600 python tools/spgemm_phases.py C1 C2 C4 C5 > $D/phases.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_C4.csv python tools/run_op.py spgemm C4 > $D/ncu.log 2>&1
