set -x
D=gpurun_out/fused2
mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/build.log 2>&1; echo build $?
timeout 1200 python -m pytest tests/test_gpu_spadd.py tests/test_gpu_setops.py tests/test_abi.py -q > $D/tests.log 2>&1; echo tests $?
timeout 600 python tools/setops_bench.py > $D/setops.txt 2>&1; echo setops $?
CSR=C3 timeout 600 python tools/probe/gather_probe.py > $D/gather_c3.txt 2>&1; echo probe $?
CSR=C5 timeout 600 python tools/probe/gather_probe.py > $D/gather_c5.txt 2>&1; echo probe5 $?
timeout 1500 python bench.py > $D/bench.log 2>&1; echo bench $?
