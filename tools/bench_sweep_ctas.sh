#!/bin/bash
# bench.py at several copy-kernel variants / CTA counts; prints value + per-launch time
for v in "$@"; do
  set -- ${v/@/ }
  GR_COPY=$1 GR_CTAS=${2:-0} timeout 120 python bench.py --no-cpu-baseline --steps 100 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', '${2:-0}', round(d['value']), round(d['roofline']['avg_launch_us'],2), round(d['roofline']['frac'],3), round(d['host_us_per_request'],2), d['latency_us']['p50'])"
done
