set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_setops.py -x -q > gpurun_out/gputests_setops.log 2>&1; echo tests $?
timeout 900 python tools/setops_bench.py gpurun_out/setops_bench.json > gpurun_out/setops_bench.log 2>&1; echo bench $?
