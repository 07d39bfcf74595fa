D=gpurun_out/scansweep2; mkdir -p $D
python tools/spgemm_phases.py C2 C5 --reps 3 > $D/p.txt 2>&1
for it in 4 6 8 12; do
MSP_BUILD_DIR=/tmp/bs$it MSP_LIB_OUT=/tmp/libs$it.so MSP_NVCC_EXTRA="-DMSP_SCAN_ITEMS=$it" python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b$it.log 2>&1
echo "== items $it" >> $D/p.txt
MSP_LIB=/tmp/libs$it.so python tools/spgemm_phases.py C2 C5 --reps 3 >> $D/p.txt 2>&1
done
