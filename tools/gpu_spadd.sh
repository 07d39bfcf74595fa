set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "spadd" > gpurun_out/gputests_spadd.log 2>&1; echo tests $?
python tools/exp/spadd_time.py C3 > gpurun_out/spadd_staged.log 2>&1
python tools/exp/spadd_time.py C2 >> gpurun_out/spadd_staged.log 2>&1
