# TMA-store epilogue: GEMM tests, the parity suite, then BERT-base A/B (mode 15 = LSU stores, 1 = TMA stores)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_gemm.py -q -x 2>&1 | tail -2
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x 2>&1 | tail -2
for m in 15 1 15 1; do
  timeout 600 python bench.py --no-baselines --no-cpu-baseline --gemm-mode $m > gpurun_out/ab_tma_$m.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/ab_tma_$m.json').read().strip().splitlines()[-1]); print('mode $m', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'], 'frac', round(d['roofline']['frac'],3))"
done
