set -x
D=gpurun_out/final5; mkdir -p $D
python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1; echo smoke $?
timeout 1800 python -m pytest tests -m gpu -q > $D/gputests.log 2>&1; echo tests $?
timeout 900 python bench.py > $D/bench.log 2>&1; echo bench $?
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $D/launches_bench.csv python bench.py --steps 1 --warmup 3 --spmv-reps 2 --no-e2e --no-cpu --no-table > $D/bench_ncu.log 2>&1; echo ncu $?
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $D/bench_ref.log 2>&1; echo ref $?
