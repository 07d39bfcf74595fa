set -x
mkdir -p gpurun_out/v1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v1/smoke.log 2>&1; echo smoke $?
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/v1/gputests.log 2>&1; echo tests $?
timeout 900 python bench.py > gpurun_out/v1/bench.log 2>&1; echo bench $?
