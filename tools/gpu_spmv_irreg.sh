# SpMV on the irregular configs: launch-shape sweep + one ncu --set full per config
set -x
mkdir -p gpurun_out
for c in C3 C4 C5; do
  timeout 900 python tools/spmv_tune.py $c "CFG=-1" "CFG=0" "CFG=-1,K=7" "CFG=-1,NW=4" >> gpurun_out/tune_irreg.log 2>&1
done
for c in C3 C4 C5; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -o gpurun_out/spmv_$c -f python tools/run_op.py spmv $c > gpurun_out/ncu_spmv_$c.log 2>&1
done
