set -x
mkdir -p gpurun_out/ncu
N="ncu --set full --clock-control none --import-source on -k regex:gemm_tile -c 2 -f"
timeout 900 $N -o /tmp/gemm_C2 python tools/run_op.py spgemm C2 > gpurun_out/ncu/gemm.log 2>&1
bash tools/ncu_digest.sh /tmp/gemm_C2.ncu-rep gpurun_out/ncu/gemm_C2
