#!/bin/bash
# bench configs under launch-time knobs: tools/env_sweep_cfg.sh "cfg1 cfg2" "ENV=.." ...
CFGS=$1; shift
for c in $CFGS; do
  for E in "$@"; do
    env $E timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/e.json 2>/dev/null
    python -c "import json; d=json.load(open('/tmp/e.json')); print('$c $E', round(d['roofline']['kernel_ms_avg'],3), round(d['ms_per_step'],3))"
  done
done
