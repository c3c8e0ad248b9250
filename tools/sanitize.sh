#!/bin/bash
# compute-sanitizer over tests/harness/sanitize.py for several copy engines; one summary line per run
mkdir -p gpurun_out/san
# the product library must match the sources (sanitize.py only loads it)
python -c "from paper_conf_eurosys_wulywdyfwwj26_b200 import _build; _build.build()" || exit 1
for eng in ${ENGINES:-default ldst8 tmas4 wv8}; do
  for tool in memcheck racecheck synccheck; do
    # "default": the product engine choice and the fast paths (GR_COPY unset)
    if [ $eng = default ]; then E="env -u GR_COPY"; else E="env GR_COPY=$eng"; fi
    $E timeout 900 compute-sanitizer --tool $tool --target-processes all python tests/harness/sanitize.py \
      > gpurun_out/san/$eng.$tool.log 2>&1
    echo "$eng $tool: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san/$eng.$tool.log | tail -1) | $(grep -c 'sanitize workload OK' gpurun_out/san/$eng.$tool.log) ok"
  done
done
