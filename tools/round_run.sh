#!/bin/bash
# Round-end measurement batch on one B200 (run under gpurun): bench line (N=1),
# reference arm, an N=2 plumbing run on one GPU, ncu launch list + full capture
# + steady traffic of gr_copy, workflows (cfg4/cfg5, interleaved cfg5 incl. 1%).
set -x
D=gpurun_out/final
mkdir -p $D
timeout 600 python bench.py > $D/bench.json 2> $D/bench.err
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > $D/ref.json 2> $D/ref.err
GR_BENCH_SAME_GPU=1 GR_BENCH_BACKEND=gloo timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 10 --no-multipath-probe > $D/bench_n2.json 2> $D/bench_n2.err
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-sweep --lat-samples 20 --e2e-steps 2 --b2b-steps 20"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file $D/launches.csv $B > $D/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gr_copy -s 60 -c 3 -o $D/full $B > $D/ncu_full.log 2>&1
ncu -i $D/full.ncu-rep --page raw --csv > $D/full_raw.csv 2>&1
timeout 600 ncu --cache-control none --clock-control none --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
  -k regex:gr_copy -s 200 -c 20 --csv --log-file $D/steady.csv $B > $D/ncu_steady.log 2>&1
timeout 1500 python tests/harness/workflows.py $D/cfg5i.json cfg5i > $D/cfg5i.log 2>&1
timeout 900 python tests/harness/workflows.py $D/workflows.json > $D/workflows.log 2>&1
# NVLink evidence when the box has two or more GPUs (in-round gpurun has one)
if [ "$(nvidia-smi -L | wc -l)" -ge 2 ]; then bash tools/ncu_nvlink.sh; fi
tail -c 300 $D/bench.json
