# round evidence: smoke, GPU tests, bench line, five-config sweep, launch list
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo tests $?
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo bench $?
timeout 1500 python tools/sweep.py --out gpurun_out/sweep.json > gpurun_out/sweep.log 2>&1; echo sweep $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --spmv-reps 2 --no-e2e --no-cpu > gpurun_out/bench_ncu.log 2>&1; echo ncu $?
