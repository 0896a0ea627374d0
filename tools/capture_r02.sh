#!/bin/bash
# Round-2 evidence on one B200 (through gpurun):  tools/capture_r02.sh TAG
TAG=${1:?tag}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest=$?; tail -3 gpurun_out/${TAG}_pytest.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo bench=$?
for c in dense africa int16 periods; do
  timeout 600 python bench.py --config $c --steps 10 > gpurun_out/${TAG}_$c.json 2> gpurun_out/${TAG}_$c.err; echo $c=$?
done
timeout 900 python bench.py --config stream --steps 8 --warmup 2 --no-cpu-baseline > gpurun_out/${TAG}_stream.json 2> gpurun_out/${TAG}_stream.err; echo stream=$?
timeout 600 python tools/periods_exp.py > gpurun_out/${TAG}_periods_exp.log 2>&1; echo pexp=$?
timeout 900 python bench.py --config sentinel2 --steps 3 --warmup 3 > gpurun_out/${TAG}_s2.json 2> gpurun_out/${TAG}_s2.err; echo s2=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"monitor|refit" -c 20 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
  > /dev/null 2>&1; echo launches=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:monitor_fused -s 3 -c 1 \
  -o gpurun_out/${TAG}_full python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
  > gpurun_out/${TAG}_ncu.log 2>&1; echo full=$?
timeout 1500 python tools/sweep_table.py gpurun_out/${TAG}_sweep.json > gpurun_out/${TAG}_sweep.log 2>&1; echo sweep=$?
