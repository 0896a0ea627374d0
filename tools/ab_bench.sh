#!/bin/bash
# A/B timing of several builds of libbfast.so on the same box, interleaved
# round-robin (R rounds):   R=2 tools/ab_bench.sh ab/a.so ab/b.so ...
# ("pkg" = the package's own build; "lib:sy,nop,per_sm" forces a TC smem layout).  Extra bench.py args via BENCH_ARGS.
# prints one line per run: <lib> <value Mpx/s> <kernel ms> <sm MHz>
R=${R:-2}
mkdir -p gpurun_out
for i in $(seq 1 $R); do
  for LL in "$@"; do
    L=${LL%%:*}; LAY=""; [ "$L" != "$LL" ] && LAY=${LL#*:}
    [ "$L" = pkg ] && L=$(pwd)/paper_conf_icde_giesekerhvo20_b200/libbfast.so
    BFAST_TC_LAYOUT=$LAY BFAST_LIB=$L timeout 600 python bench.py --no-e2e --no-cpu-baseline $BENCH_ARGS > gpurun_out/ab.json 2> gpurun_out/ab.err
    python -c "
import json,sys; d=json.load(open('gpurun_out/ab.json'))
ps=d.get('parity_sample') or {}
print('$(basename $L):$LAY', round(d['value']/1e6,1), round(d['roofline']['kernel_ms_avg'],3), d['clocks']['sm_mhz'],
      'parity', ps.get('ok'), ps.get('break_mismatch'), ps.get('mag_max_scaled_err'))" || tail -3 gpurun_out/ab.err
  done
done
