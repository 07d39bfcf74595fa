D=gpurun_out/gsweep; mkdir -p $D
python tools/spgemm_phases.py C2 C5 --reps 3 > $D/p.txt 2>&1
for cfg in "4 8 3 4" "16 8 3 4" "8 4 6 4" "8 16 1 4" "8 8 3 2" "8 8 3 8"; do
set -- $cfg
n=$1_$2_$3_$4
MSP_BUILD_DIR=/tmp/bg$n MSP_LIB_OUT=/tmp/libg$n.so MSP_NVCC_EXTRA="-DMSP_WR_SYM_WARPS=$1 -DMSP_WR_NUM_WARPS=$2 -DMSP_WR_NUM_MINB=$3 -DMSP_WS_WARPS=$4" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$n.log 2>&1
echo "== sym $1 num $2 minb $3 ws $4" >> $D/p.txt
MSP_LIB=/tmp/libg$n.so python tools/spgemm_phases.py C2 C5 --reps 3 >> $D/p.txt 2>&1
done
