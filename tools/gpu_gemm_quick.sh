# SpGEMM GPU tests, bench line (SpGEMM ms beside SpMV), ncu --set full of the C2 tile kernels (digest only)
set -x
mkdir -p gpurun_out/ncu
timeout 900 python -m pytest tests -m gpu -x -q -k "spgemm" > gpurun_out/gputests_spgemm.log 2>&1; echo tests $?
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_gemm.log 2>&1; echo bench $?
if [ -n "$NCU" ]; then bash tools/gpu_ncu_gemm.sh; fi
