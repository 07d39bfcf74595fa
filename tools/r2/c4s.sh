D=gpurun_out/c4s; mkdir -p $D
python paper_conf_ipps_daltonbmog15_b200/_build.py > $D/b.log 2>&1
python tools/spmv_tune.py C4 "VERBOSE=1" "CFG=12" "CFG=13" "CFG=14" "CFG=15" > $D/tune.txt 2>&1
python tools/spmv_tune.py C1 "VERBOSE=1" "CFG=12" "CFG=14" >> $D/tune.txt 2>&1
