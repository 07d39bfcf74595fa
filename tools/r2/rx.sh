set -x
D=gpurun_out/${RX_DIR:-rx2}
mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_spgemm_radix.py -x -q > $D/tests.log 2>&1; echo tests $?
python tools/spgemm_compare.py C1 C2 C4 --json $D/compare.json > $D/compare.txt 2>&1
for bits in 0 28; do for two in 0 1; do
MSP_RX_SORT_BITS=$bits MSP_RX_TWO_PASS=$two python tools/spgemm_compare.py C1 > $D/fig4_b${bits}_t${two}.txt 2>&1
done; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 80 --csv python tools/spgemm_compare.py C2:0.3 > $D/launches_c2.csv 2>&1
