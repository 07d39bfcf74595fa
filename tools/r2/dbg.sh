D=gpurun_out/dbg; mkdir -p $D
timeout 300 compute-sanitizer --tool memcheck python tools/r2/dbg_small.py 3000 > $D/m1.txt 2>&1; echo $?
timeout 300 python tools/r2/dbg_small.py 300000 > $D/m2.txt 2>&1; echo $?
