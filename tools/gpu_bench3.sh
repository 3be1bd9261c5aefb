# three default bench runs back to back (run-to-run spread of the headline)
for i in 1 2 3; do
  timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/bench3_$i.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/bench3_$i.json').read().strip().splitlines()[-1]); print('BB', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])"
done
