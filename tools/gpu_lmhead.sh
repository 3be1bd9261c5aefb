timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_dp.py -q -x -k "gpt2 or lm or g2" 2>&1 | tail -2
for i in 1 2; do
  timeout 600 python bench.py --config gpt2-medium --steps 30 --no-baselines --no-cpu-baseline > gpurun_out/lm.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/lm.json').read().strip().splitlines()[-1]); print('gpt2', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])"
done
