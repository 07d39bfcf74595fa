# set-operation tests at the default build, then the Fig 2 sweep per items-per-thread build
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_setops.py -x -q > gpurun_out/gputests_setops.log 2>&1; echo tests $?
timeout 900 python tools/setops_bench.py gpurun_out/setops_bench.json > gpurun_out/setops_bench.log 2>&1; echo bench $?
for ipt in ${IPTS:-8 16}; do
  touch paper_conf_ipps_daltonbmog15_b200/csrc/setops.cu; MSP_NVCC_EXTRA="-DMSP_SET_IPT=$ipt" timeout 300 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_ipt$ipt.log 2>&1
  timeout 900 python tools/setops_bench.py gpurun_out/setops_bench_ipt$ipt.json > gpurun_out/setops_bench_ipt$ipt.log 2>&1; echo bench$ipt $?
done
