mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'share', round(d['roofline']['share_of_step'],3), 'rr', d.get('recompute_ratio'), d['clocks']['sm_mhz'])" 2>&1 | tail -1; }
for c in roberta-large bert-large gpt2-medium; do
  timeout 600 python bench.py --config $c --steps 30 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; echo "$c rc=$? $(summ gpurun_out/bench_$c.log)"
done
timeout 300 python bench.py --no-cpu-baseline --no-baselines > gpurun_out/bench_d.log 2>&1; echo "bb: $(summ gpurun_out/bench_d.log)"
