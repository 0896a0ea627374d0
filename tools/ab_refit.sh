mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/ab_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/ab_tests.log
for i in 1 2; do for L in a b; do
BFAST_LIB=$PWD/ab/$L.so timeout 300 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/ab_$L.json 2>gpurun_out/ab_$L.err
python -c "
import json; d=json.load(open('gpurun_out/ab_$L.json')); ps=d['parity_sample']
print('$L', round(d['value']/1e6,1), 'step', round(d['ms_per_step'],3), 'kern', round(d['roofline']['kernel_ms_avg'],3), d['clocks']['sm_mhz'], ps['ok'], ps['break_mismatch'], ps['mag_max_scaled_err'])" || tail -3 gpurun_out/ab_$L.err
done; done
BFAST_LIB=$PWD/ab/b.so timeout 300 ncu --set full --clock-control none --import-source on -k regex:refit -s 1 -c 1 -o gpurun_out/refit_full_b python tools/refit_probe.py > gpurun_out/rp_ncu_b.log 2>&1; echo ncu=$?
