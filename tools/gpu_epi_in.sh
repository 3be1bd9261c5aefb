# coalesced epilogue inputs: GEMM tests, microbench of the input epilogues, BERT-base bench x2
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_gemm.py -q -x 2>&1 | tail -2
for shp in "5376 3072 768" "5376 768 3072" "5376 768 768"; do
  for e in 3 4 5 10; do for m in 15 1; do python tools/one_gemm.py $m $e $shp 0 0 20 2>&1 | grep TFLOP; done; done
done
for i in 1 2; do
  timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/epi_in_$i.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/epi_in_$i.json').read().strip().splitlines()[-1]); print('bench', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'], 'frac', round(d['roofline']['frac'],3))"
done
