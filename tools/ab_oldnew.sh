for cfg in sweep:100:0.1:1 sweep:100:0.1:3 sweep:1000:0.1:5 landsat; do
  for r in 1 2; do
    for side in new old; do
      if [ $side = old ]; then D=ab/oldrepo; else D=.; fi
      (cd $D && timeout 300 python bench.py --config $cfg --steps 10 --no-e2e --no-cpu-baseline > /tmp/o.json 2>/tmp/o.err; python -c "import json; d=json.load(open('/tmp/o.json')); print('$cfg $side', round(d['ms_per_step'],3), round(d['roofline']['kernel_ms_avg'],3))" || tail -2 /tmp/o.err)
    done
  done
done
