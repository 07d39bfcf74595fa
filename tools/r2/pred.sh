D=gpurun_out/pred; mkdir -p $D
timeout 2400 python tools/predict_sweep.py --json $D/predictability_sweep.json > $D/log.txt 2>&1; echo p $?
