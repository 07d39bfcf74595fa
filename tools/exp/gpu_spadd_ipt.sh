# SpAdd items-per-thread sweep: one experiment build per IPT, C3 and C2 timed
set -x
mkdir -p gpurun_out
for ipt in ${IPTS:-8 10 12 16}; do
  touch paper_conf_ipps_daltonbmog15_b200/csrc/spadd.cu
  MSP_NVCC_EXTRA="-DMSP_ADD_IPT=$ipt" python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_add_ipt$ipt.log 2>&1
  for c in C3 C2; do echo "ipt=$ipt" >> gpurun_out/spadd_ipt.log; python tools/exp/spadd_time.py $c >> gpurun_out/spadd_ipt.log 2>&1; done
done
