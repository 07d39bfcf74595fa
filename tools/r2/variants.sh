# build libmsp variants (macro sets) side by side and time SpMV on C2 with each
set -x
D=gpurun_out/${VAR_DIR:-variants}
mkdir -p $D
i=0
for v in "$@"; do
  i=$((i+1))
  MSP_NVCC_EXTRA="$v" MSP_BUILD_DIR=/tmp/msp_b$i MSP_LIB_OUT=/tmp/libmsp_$i.so python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build_$i.log 2>&1 &
done
wait
i=0
for v in "$@"; do
  i=$((i+1))
  echo "== variant $i: $v" >> $D/tune.txt
  MSP_LIB=/tmp/libmsp_$i.so python tools/spmv_tune.py ${CFGS:-C2} "CFG=-3" "CFG=-3" >> $D/tune.txt 2>&1
done
