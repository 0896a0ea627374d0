#!/bin/bash
# A/B of fp64-refit builds on one box (run through gpurun):
#   tools/ab_refit.sh ab/b.so ab/c.so ...
# per lib: the refit kernel's launch durations (ncu, clock-control none)
# and the whole call (refit_probe.py, CUDA events)
mkdir -p gpurun_out
for L in "$@"; do
  n=$(basename $L .so)
  BFAST_LIB=$PWD/$L timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:refit -c 6 --csv \
    --log-file gpurun_out/abr_$n.csv python tools/refit_probe.py > gpurun_out/abr_$n.log 2>&1
  python - "$n" <<'PY'
import csv, sys
n = sys.argv[1]
rows = [r for r in csv.reader(open(f"gpurun_out/abr_{n}.csv")) if len(r) > 10 and r[-3] == "gpu__time_duration.sum"]
print(n, "refit us", [r[-1] for r in rows])
PY
  BFAST_LIB=$PWD/$L timeout 300 python tools/refit_probe.py | tail -1
done
