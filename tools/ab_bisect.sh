#!/bin/bash
# Bench one config in several repository snapshots, interleaved (GPU box):
#   tools/ab_bisect.sh CFG dir1 dir2 ...     ("." = this tree)
# A snapshot dir holds bench.py, oracle/, include/, MEASURED_PEAKS.json and the
# package with its built libbfast.so (e.g. from a git worktree of an older
# commit, copied under ab/, which gpurun ships and git ignores).
CFG=$1; shift
for r in 1 2; do
  for D in "$@"; do
    (cd $D && timeout 300 python bench.py --config $CFG --steps 10 --no-e2e --no-cpu-baseline > /tmp/o.json 2>/tmp/o.err; python -c "import json; d=json.load(open('/tmp/o.json')); print('$CFG $D', round(d['ms_per_step'],3), round(d['roofline']['kernel_ms_avg'],3))" || tail -2 /tmp/o.err)
  done
done
