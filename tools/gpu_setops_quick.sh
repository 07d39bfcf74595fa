# set-operation tests (default build and a forced two-walk build), Fig 2 sweep, launch list at 1e8 keys-32 union
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_setops.py -x -q > gpurun_out/gputests_setops.log 2>&1; echo tests $?
timeout 900 python tools/setops_bench.py gpurun_out/setops_bench.json > gpurun_out/setops_bench.log 2>&1; echo bench $?
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/setops_launches.csv python tools/run_setop.py union keys-32 100000000 3 > gpurun_out/setops_ncu1.log 2>&1; echo list $?
if [ -n "$FULL" ]; then timeout 600 ncu --set full --clock-control none --import-source on -k regex:set_tile_kernel -s 2 -c 1 -o gpurun_out/setops_tile -f python tools/run_setop.py union keys-32 100000000 3 > gpurun_out/setops_ncu2.log 2>&1; echo full $?; fi
if [ -n "$WALK2" ]; then
  touch paper_conf_ipps_daltonbmog15_b200/csrc/setops.cu
  MSP_NVCC_EXTRA="-DMSP_SET_FORCE_WALK2" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_set_walk2.log 2>&1
  timeout 900 python -m pytest tests/test_gpu_setops.py -x -q > gpurun_out/gputests_setops_walk2.log 2>&1; echo tests_walk2 $?
fi
