set -x
mkdir -p gpurun_out/ncu
N="ncu --set full --clock-control none --import-source on -k regex:spmv -c 1 -f"
run() { name=$1; shift; env "$@" timeout 600 $N -o /tmp/$name python tools/run_op.py spmv ${name##*_} >> gpurun_out/ncu/ncu.log 2>&1; bash tools/ncu_digest.sh /tmp/$name.ncu-rep gpurun_out/ncu/$name; }
run mp_C2 MSP_SPMV_CFG=-2
run rowk_C2 MSP_SPMV_CFG=-1
run mpst3_C2 MSP_SPMV_CFG=-2 MSP_SPMV_ST=3 MSP_SPMV_K=21
run mp_C3 MSP_SPMV_CFG=-2
run tr_C3 MSP_SPMV_CFG=0
ls -la gpurun_out/ncu
