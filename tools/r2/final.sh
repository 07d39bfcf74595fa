# end-of-round evidence (round 2): smoke, all GPU tests, bench line, SpMV ncu
# (launch list + --set full), sanitizers, ablations
set -x
D=gpurun_out/final
mkdir -p $D
python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1; echo smoke $?
timeout 2400 python -m pytest tests -m gpu -q > $D/gputests.log 2>&1; echo tests $?
timeout 1200 python bench.py > $D/bench.log 2>&1; echo bench $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/launches.csv python bench.py --steps 1 --warmup 3 --spmv-reps 2 --no-e2e --no-cpu --no-table > $D/bench_ncu.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_wt -c 1 -f -o /tmp/spmv_C2 python tools/run_op.py spmv C2 > $D/ncu_full.log 2>&1
ncu -i /tmp/spmv_C2.ncu-rep --page raw --csv > $D/spmv_C2_raw.csv 2>/dev/null
ncu -i /tmp/spmv_C2.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | python tools/ncu_lines.py 60 > $D/spmv_C2_lines.txt
for tool in memcheck synccheck initcheck racecheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 200 python tools/sanitize_cases.py > $D/sanitize_$tool.txt 2>&1; echo $tool $?
done
python tools/dense_spgemm.py 1000 2000 > $D/dense.txt 2>&1
MSP_SPGEMM_SEGMENTED=0 python tools/dense_spgemm.py 1000 > $D/dense_esc.txt 2>&1
for c in C1 C2 C3 C4 C5; do python tools/spmv_tune.py $c "VERBOSE=1" >> $D/spmv_default_tune.txt 2>&1; done
timeout 600 python tools/setops_bench.py > $D/setops.txt 2>&1; echo setops $?
