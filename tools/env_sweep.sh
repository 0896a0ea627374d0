#!/bin/bash
# Landsat bench under launch-time knobs (no rebuild): tools/env_sweep.sh "ENV=.. ENV2=.." ...
for r in 1 2; do
  for E in "$@"; do
    env $E timeout 300 python bench.py --steps 10 --no-e2e --no-cpu-baseline > /tmp/e.json 2>/dev/null
    python -c "import json; d=json.load(open('/tmp/e.json')); print('$E', round(d['roofline']['kernel_ms_avg'],3), round(d['ms_per_step'],3))"
  done
done
