set -x
D=gpurun_out/fig4
mkdir -p $D
for bits in 0 28; do for two in 0 1; do
MSP_RX_SORT_BITS=$bits MSP_RX_TWO_PASS=$two python tools/fig4_probe.py 5 > $D/events_b${bits}_t${two}.txt 2>&1
MSP_RX_SORT_BITS=$bits MSP_RX_TWO_PASS=$two timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum --clock-control none -k regex:rx_tile -c 3 --csv --log-file $D/ncu_b${bits}_t${two}.csv python tools/fig4_probe.py 2 > /dev/null 2>&1
done; done
