set -x
mkdir -p gpurun_out/off
timeout 400 python bench.py > gpurun_out/off/bench.json 2> gpurun_out/off/bench.err
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/off/ref.json 2> gpurun_out/off/ref.err
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/off/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/off/ncu_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gr_copy -s 60 -c 3 -o gpurun_out/off/full python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/off/ncu_full.log 2>&1
ncu -i gpurun_out/off/full.ncu-rep --page raw --csv > gpurun_out/off/full_raw.csv 2>&1
tail -c 600 gpurun_out/off/bench.json
