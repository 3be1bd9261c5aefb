mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'rr', d.get('recompute_ratio'), d['clocks'])" 2>&1 | tail -1; }
for cfg in "0 0" "1 0" "1 1"; do set -- $cfg
  MIMOSE_PDL=$1 MIMOSE_WGRAD_FUSED=$2 timeout 300 python bench.py --no-cpu-baseline --no-baselines > gpurun_out/bench_p$1_f$2.log 2>&1
  echo "pdl=$1 fused=$2: $(summ gpurun_out/bench_p$1_f$2.log)"
done
timeout 600 python bench.py > gpurun_out/bench_full.log 2>&1; echo "full: $(summ gpurun_out/bench_full.log)"
for c in bert-large roberta-large gpt2-medium; do
  timeout 600 python bench.py --config $c --steps 30 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; echo "$c rc=$? $(summ gpurun_out/bench_$c.log)"
done
