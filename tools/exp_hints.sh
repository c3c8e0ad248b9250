# copy-engine experiments: L2 prefetch ahead inside the loop, large sizes
mkdir -p gpurun_out/exp4
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "variants and PFLOOP" > gpurun_out/exp4/tests.txt 2>&1
timeout 300 python tools/copybench.py torch tma8 > gpurun_out/exp4/cb.txt 2>&1
for cfg in "GR_PF=1" "GR_PF=1 GR_PFLOOP=1" "GR_PF=2 GR_PFLOOP=1" "GR_PF=4 GR_PFLOOP=1" "GR_PF=8 GR_PFLOOP=1"; do
  echo "== $cfg" >> gpurun_out/exp4/cb.txt
  env $cfg timeout 300 python tools/copybench.py wv8 wv4 >> gpurun_out/exp4/cb.txt 2>&1
done
bash tools/bench_env.sh GR_COPY=wv8,GR_PF=1 GR_COPY=wv8,GR_PF=1,GR_PFLOOP=1 GR_COPY=wv8,GR_PF=2,GR_PFLOOP=1 GR_COPY=wv4,GR_PF=1,GR_PFLOOP=1 > gpurun_out/exp4/env.txt 2>&1
tail -2 gpurun_out/exp4/tests.txt; cat gpurun_out/exp4/cb.txt gpurun_out/exp4/env.txt
