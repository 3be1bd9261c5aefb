# CTA-pair A/B inside the step: BERT-large and GPT-2 medium (mode 17 = pair for every split-1 N%256 GEMM)
for spec in "8192 4096 1024 0 0" "8192 1024 4096 0 0"; do
  for e in 2 3 8 10; do for m in 1 17; do timeout 60 python tools/one_gemm.py $m $e $spec 20 2>&1 | grep TFLOP; done; done
done
for c in bert-large gpt2-medium; do for m in 1 17 1 17; do
  timeout 600 python bench.py --config $c --steps 30 --no-baselines --no-cpu-baseline --gemm-mode $m > gpurun_out/p3.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/p3.json').read().strip().splitlines()[-1]); print('$c mode $m', round(d['value'],1), round(d['ms_per_step'],3), d['clocks']['sm_mhz'])"
done; done
