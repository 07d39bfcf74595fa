# round-2 baseline on a fresh box: smoke, GPU tests, bench, SpMV C2 ncu (source lines) for 1 and 2 CTAs/SM
set -x
mkdir -p gpurun_out/r2base
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2base/smoke.log 2>&1; echo smoke $?
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2base/gputests.log 2>&1; echo tests $?
timeout 600 python bench.py --no-cpu > gpurun_out/r2base/bench.log 2>&1; echo bench $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -f -o /tmp/spmv_C2 python tools/run_op.py spmv C2 > gpurun_out/r2base/ncu1.log 2>&1
ncu -i /tmp/spmv_C2.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 80 > gpurun_out/r2base/spmv_C2_lines.txt
ncu -i /tmp/spmv_C2.ncu-rep --page raw --csv > gpurun_out/r2base/spmv_C2_raw.csv 2>/dev/null
ncu -i /tmp/spmv_C2.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | gzip > gpurun_out/r2base/spmv_C2_source.csv.gz
MSP_SPMV_NW=4 timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -f -o /tmp/spmv_C2_nw4 python tools/run_op.py spmv C2 > gpurun_out/r2base/ncu2.log 2>&1
ncu -i /tmp/spmv_C2_nw4.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 80 > gpurun_out/r2base/spmv_C2_nw4_lines.txt
ncu -i /tmp/spmv_C2_nw4.ncu-rep --page raw --csv > gpurun_out/r2base/spmv_C2_nw4_raw.csv 2>/dev/null
