set -x
D=gpurun_out/gprobe
mkdir -p $D
python tools/probe/gather_probe.py 20 23 26 27 > $D/probe.txt 2>&1
REPS=1 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,gpu__time_duration.sum --clock-control none -k regex:gather4 --csv --log-file $D/ncu27.csv python tools/probe/gather_probe.py 27 > $D/ncu27.log 2>&1
