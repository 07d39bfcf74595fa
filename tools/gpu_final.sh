# end-of-round evidence: smoke, all GPU tests, bench line, sweep, launch list, SpMV ncu capture
set -x
mkdir -p gpurun_out/ncu
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gputests.log 2>&1; echo tests $?
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo bench $?
timeout 1500 python tools/sweep.py --out gpurun_out/sweep.json > gpurun_out/sweep.log 2>&1; echo sweep $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --spmv-reps 2 --no-e2e --no-cpu > gpurun_out/bench_ncu.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_merge -c 1 -f -o /tmp/spmv_C2 python tools/run_op.py spmv C2 > gpurun_out/ncu/spmv.log 2>&1
bash tools/ncu_digest.sh /tmp/spmv_C2.ncu-rep gpurun_out/ncu/spmv_C2_final
timeout 600 python tools/setops_bench.py gpurun_out/setops_bench.json > gpurun_out/setops_bench.log 2>&1; echo setops $?
