#!/bin/bash
# Round-end measurement batch on one B200 (run under gpurun): bench line, reference arm,
# ncu launch list + full capture of gr_copy, cfg3 sweep, ablation, workflows.
set -x
D=gpurun_out/final
mkdir -p $D
timeout 400 python bench.py > $D/bench.json 2> $D/bench.err
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > $D/ref.json 2> $D/ref.err
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $D/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $D/ncu_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gr_copy -s 60 -c 3 -o $D/full python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $D/ncu_full.log 2>&1
ncu -i $D/full.ncu-rep --page raw --csv > $D/full_raw.csv 2>&1
timeout 900 python tests/harness/sweep.py $D/sweep.json > $D/sweep.log 2>&1
timeout 600 python tools/ablation.py $D/ablation.json > $D/ablation.log 2>&1
timeout 900 python tests/harness/workflows.py $D/workflows.json > $D/workflows.log 2>&1
timeout 600 python tests/harness/workflows.py $D/cfg2.json cfg2 > $D/cfg2.log 2>&1
timeout 900 python tests/harness/workflows.py $D/cfg5i.json cfg5i > $D/cfg5i.log 2>&1
tail -c 300 $D/bench.json
