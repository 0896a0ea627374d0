#!/bin/bash
# Round evidence on one B200 (run through gpurun):   tools/capture_evidence.sh TAG
#   gpurun_out/TAG_bench.json      default bench line (landsat, e2e, cpu baseline)
#   gpurun_out/TAG_s2.json         Sentinel-2 tile (configs[3]) slab by slab on one GPU
#   gpurun_out/TAG_stream.json     pinned-host streaming (configs[4])
#   gpurun_out/TAG_launches.csv    ncu launch list (gpu__time_duration, clock-control none)
#   gpurun_out/TAG_full.ncu-rep    ncu --set full of one monitor_fused launch
# then (here):  python profiles/summarize.py full|launches ...
TAG=${1:?tag}
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo bench=$?
timeout 900 python bench.py --config sentinel2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_s2.json 2> gpurun_out/${TAG}_s2.err; echo s2=$?
timeout 900 python bench.py --config stream --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_stream.json 2> gpurun_out/${TAG}_stream.err; echo stream=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"monitor|refit" -c 20 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
  > /dev/null 2>&1; echo launches=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:monitor_fused -s 3 -c 1 \
  -o gpurun_out/${TAG}_full python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
  > gpurun_out/${TAG}_ncu.log 2>&1; echo full=$?
