D=gpurun_out/umax; mkdir -p $D
python tools/spgemm_phases.py C2 --reps 6 > $D/p.txt 2>&1
for cfg in "256 4" "256 3" "128 4" "128 5"; do
set -- $cfg
MSP_BUILD_DIR=/tmp/bu$1$2 MSP_LIB_OUT=/tmp/libu$1$2.so MSP_NVCC_EXTRA="-DMSP_WR_UMAX=$1 -DMSP_WR_NUM_MINB=$2" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$1$2.log 2>&1
echo "== umax $1 minb $2" >> $D/p.txt
MSP_LIB=/tmp/libu$1$2.so python tools/spgemm_phases.py C2 --reps 6 >> $D/p.txt 2>&1
done
MSP_LIB=/tmp/libu2564.so timeout 900 python -m pytest tests/test_gpu_spgemm_rowacc.py -k "not esc_tile" -q > $D/tests.log 2>&1; echo t $?
