set -x
mkdir -p gpurun_out/ncu
N="ncu --set full --clock-control none --import-source on -k regex:spadd_tile -c 2 -f"
timeout 900 $N -o /tmp/spadd_C3 python tools/run_op.py spadd C3 > gpurun_out/ncu/spadd.log 2>&1
bash tools/ncu_digest.sh /tmp/spadd_C3.ncu-rep gpurun_out/ncu/spadd_C3
N="ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -f"
timeout 900 $N -o /tmp/spmv_C2 python tools/run_op.py spmv C2 > gpurun_out/ncu/spmv.log 2>&1
bash tools/ncu_digest.sh /tmp/spmv_C2.ncu-rep gpurun_out/ncu/spmv_C2
