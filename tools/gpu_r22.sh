mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'rr', d.get('recompute_ratio'), 'static', d.get('static_plan'), 'sub', d.get('sublayer_units'), d['mimose']['mean_layers_dropped'], d['clocks'])"
for c in bert-large roberta-large; do
timeout 900 python bench.py --config $c --steps 30 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; echo "$c rc=$?"
tail -1 gpurun_out/bench_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'rr', d.get('recompute_ratio'), 'sub', d.get('sublayer_units'), d['mimose']['mean_layers_dropped'])"
done
