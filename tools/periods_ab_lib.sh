#!/bin/bash
# f1 timing (tools/periods_exp.py, yearly sets) under several library builds:
#   tools/periods_ab_lib.sh pkg ab/x.so ...
for L in "$@"; do
  LL=$L; [ "$L" = pkg ] && LL=$(pwd)/paper_conf_icde_giesekerhvo20_b200/libbfast.so
  echo "== $L"; BFAST_LIB=$LL timeout 300 python tools/periods_exp.py 2>&1 | grep "^{" | grep yearly
done
