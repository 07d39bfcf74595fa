set -x
D=gpurun_out/${SA_DIR:-spadd1}
mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spadd.py tests/test_gpu_fullsize.py -k "spadd or c3_spadd" -x -q > $D/tests.log 2>&1; echo tests $?
python tools/spadd_phases.py C3 > $D/c3.txt 2>&1
python tools/spadd_phases.py C2 > $D/c2.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:spadd -c 6 --csv python tools/spadd_phases.py C3 > $D/ncu.csv 2>&1
