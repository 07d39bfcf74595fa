set -x
D=gpurun_out/sanitize
mkdir -p $D
for tool in memcheck synccheck initcheck racecheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 200 python tools/sanitize_cases.py > $D/$tool.txt 2>&1; echo $tool $?
done
MSP_SPMV_WT=0 timeout 900 compute-sanitizer --tool racecheck --print-limit 200 python tools/sanitize_cases.py > $D/racecheck_ctatile.txt 2>&1; echo ctatile $?
