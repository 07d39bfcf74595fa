set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "spadd" > gpurun_out/gputests_spadd.log 2>&1; echo tests $?
python tools/exp/spadd_time.py C3 > gpurun_out/spadd_staged.log 2>&1
python tools/exp/spadd_time.py C2 >> gpurun_out/spadd_staged.log 2>&1
# fallback (two-walk) path of the fill kernel, forced
touch paper_conf_ipps_daltonbmog15_b200/csrc/spadd.cu
MSP_NVCC_EXTRA="-DMSP_ADD_FORCE_WALK2" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_walk2.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "spadd" > gpurun_out/gputests_spadd_walk2.log 2>&1; echo tests_walk2 $?
