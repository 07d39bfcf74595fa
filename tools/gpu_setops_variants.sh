# Fig 2 sweep per experiment build: VARIANTS="name:flags;name:flags" (flags with commas for spaces)
set -x
mkdir -p gpurun_out
IFS=';' read -ra VS <<< "$VARIANTS"
for v in "${VS[@]}"; do
  name=${v%%:*}; flags=${v#*:}; flags=${flags//,/ }
  touch paper_conf_ipps_daltonbmog15_b200/csrc/setops.cu
  MSP_NVCC_EXTRA="$flags" timeout 300 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$name.log 2>&1
  timeout 600 python -m pytest tests/test_gpu_setops.py -x -q > gpurun_out/gputests_setops_$name.log 2>&1; echo tests_$name $?
  timeout 900 python tools/setops_bench.py gpurun_out/setops_bench_$name.json > gpurun_out/setops_bench_$name.log 2>&1; echo bench_$name $?
done
