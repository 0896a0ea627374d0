#!/bin/bash
# Landsat bench for (library, env) pairs, interleaved: tools/lib_env_ab.sh "pkg|X=0" "ab/a.so|BFAST_FZ_SC=2" ...
for r in 1 2; do
  for PAIR in "$@"; do
    L=${PAIR%%|*}; E=${PAIR#*|}
    [ "$L" = pkg ] && L=$(pwd)/paper_conf_icde_giesekerhvo20_b200/libbfast.so
    env BFAST_LIB=$L $E timeout 300 python bench.py --steps 10 --no-e2e --no-cpu-baseline $BENCH_ARGS > /tmp/e.json 2>/dev/null
    python -c "import json; d=json.load(open('/tmp/e.json')); print('$PAIR', round(d['roofline']['kernel_ms_avg'],3), round(d['ms_per_step'],3))"
  done
done
