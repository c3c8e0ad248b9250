#!/bin/bash
# PCIe evidence per library call through the library's own NVTX ranges
# (SURVEY §5, §8(d)): ncu application-range replay of the "grouter_put" and
# "grouter_get" ranges of tools/ncu_pcie.py (a 256 MiB cFn put = H2D on the
# copy engine, and a cFn get of it = D2H), PCIe bytes per range.
D=gpurun_out/ncu_nvtx
mkdir -p $D
for r in grouter_put grouter_get; do
  timeout 600 ncu --replay-mode app-range --nvtx --nvtx-include "grouter@$r/" \
    --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,gpu__time_duration.sum --csv \
    --log-file $D/$r.csv python tools/ncu_pcie.py > $D/$r.log 2>&1
  echo "$r: $(grep -c pcie $D/$r.csv) metric rows"
done
