#!/bin/bash
# compute-sanitizer over tests/harness/sanitize.py for several copy engines; one summary line per run
mkdir -p gpurun_out/san
for eng in ${ENGINES:-ldst8 tmas4 wv8}; do
  for tool in memcheck racecheck synccheck; do
    GR_COPY=$eng timeout 900 compute-sanitizer --tool $tool --target-processes all python tests/harness/sanitize.py \
      > gpurun_out/san/$eng.$tool.log 2>&1
    echo "$eng $tool: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san/$eng.$tool.log | tail -1) | $(grep -c 'sanitize workload OK' gpurun_out/san/$eng.$tool.log) ok"
  done
done
