timeout 600 python -m pytest tests/test_gpu_gemm.py -q -x 2>&1 | tail -2
timeout 1200 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -q -x 2>&1 | tail -2
for c in bert-base bert-large; do
  timeout 600 python bench.py --config $c --steps 50 --no-baselines --no-cpu-baseline > gpurun_out/p4.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/p4.json').read().strip().splitlines()[-1]); print('$c', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'], round(d['roofline']['frac'],3))"
done
