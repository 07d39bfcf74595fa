set -x
D=gpurun_out/l1
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
MSP_NVCC_EXTRA="-DMSP_SPMV_GATHER=0" MSP_BUILD_DIR=/tmp/bg0 MSP_LIB_OUT=/tmp/libg0.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b0.log 2>&1
MSP_NVCC_EXTRA="-DMSP_SPMV_GATHER=4" MSP_BUILD_DIR=/tmp/bg4 MSP_LIB_OUT=/tmp/libg4.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b4.log 2>&1
for c in C3 C4 C5 C1; do
python tools/spmv_tune.py $c "VERBOSE=1" "L1=1" "L1=1,CFG=6" >> $D/tune_g3.txt 2>&1
MSP_LIB=/tmp/libg0.so python tools/spmv_tune.py $c "VERBOSE=1" "L1=1" "L1=1,CFG=6" >> $D/tune_g0.txt 2>&1
MSP_LIB=/tmp/libg4.so python tools/spmv_tune.py $c "VERBOSE=1" "L1=1" "L1=1,CFG=6" >> $D/tune_g4.txt 2>&1
done
timeout 600 python tools/setops_bench.py > $D/setops.txt 2>&1; echo setops $?
bash tools/r2/ncu_add.sh
