timeout 600 python -m pytest tests/test_gpu_gemm.py -q -x 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -2
for shp in "5376 3072 768" "8192 4096 1024"; do for e in 0 2; do python tools/one_gemm.py 1 $e $shp 0 0 20 2>&1 | grep TFLOP; done; done
for i in 1 2; do
  timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/ge.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/ge.json').read().strip().splitlines()[-1]); print('bench', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'], 'frac', round(d['roofline']['frac'],3))"
done
