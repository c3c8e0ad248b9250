#!/bin/bash
# NVLink evidence for the D2D push: needs a box with >= 2 GPUs
# (the in-round gpurun has one; the driver's multi-GPU run can call this).
# One process drives both GPUs (never wrap a multi-rank command in ncu).
D=gpurun_out/ncu_nvlink
mkdir -p $D
timeout 300 python tools/d2d_probe.py > $D/d2d_probe.json 2>&1
timeout 900 ncu --metrics nvltx__bytes_data_user.sum,nvlrx__bytes_data_user.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
  --clock-control none -k regex:gr_copy --csv --log-file $D/nvlink.csv python tools/d2d_probe.py > $D/ncu.log 2>&1
tail -3 $D/d2d_probe.json
