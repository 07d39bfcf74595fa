# set union keys-32 at 1e8 inputs: launch list, then one --set full capture of the tile kernel
set -x
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/setops_launches.csv python tools/run_setop.py union keys-32 100000000 3 > gpurun_out/setops_ncu1.log 2>&1; echo list $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:set_tile_kernel -s 2 -c 1 -o gpurun_out/setops_tile python tools/run_setop.py union keys-32 100000000 3 > gpurun_out/setops_ncu2.log 2>&1; echo full $?
