#!/bin/bash
# bench.py under several env settings: "NAME=VAL,NAME=VAL" ...; prints value, µs/launch, frac, host µs, p50
for e in "$@"; do
  env $(echo $e | tr ',' ' ') timeout 120 python bench.py --no-cpu-baseline --steps 100 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$e', round(d['value']), round(d['roofline']['avg_launch_us'],2), round(d['roofline']['frac'],3), round(d['host_us_per_request'],2), d['latency_us']['p50'])"
done
