set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "spgemm" > gpurun_out/gputests_spgemm.log 2>&1; echo tests $?
