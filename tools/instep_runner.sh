#!/bin/bash
# runs tools/instep.py scenarios in separate processes with timeouts (a hang kills only its case)
for cfg in "PROF" "PROF GR_NO_GATE=1" "PROF GR_NO_FAST=1"; do
  echo "=== $cfg"
  env $(echo $cfg | sed 's/PROF//') timeout 90 python tools/instep.py 2>&1 | tail -25
  echo "rc=$?"
done
